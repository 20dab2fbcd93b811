"""Segment-table tile layout on CPU: builds tests/tile_check.cpp against the
library's own tables.h (seg_layout: the executor's per-VP layout; tile_range: the function
the sm_100a kernels call) and checks, over random and adversarial sizes, every start
misalignment and element size, that a VP's tiles partition [0, n) exactly with every
vector-path tile whole and 16-B aligned."""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))


def test_tiles_partition_every_vp_exactly(tmp_path):
    exe = tmp_path / "tile_check"
    subprocess.run(["g++", "-O1", "-std=c++17", "-Wall", "-o", str(exe), os.path.join(HERE, "tile_check.cpp")],
                   check=True, capture_output=True, text=True)
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0 and r.stdout.startswith("OK"), r.stdout + r.stderr
