#!/bin/bash
# Host sanitizers for the C++ core: build the host sources of libsvp with
# ASan+UBSan and, separately, TSan (the guest-kernel objects are the normal nvcc ones), then
# run the CPU test suite's library tests against each build in dry-run contexts (no GPU:
# planner, dispatcher, VP Control threads, IPC server thread + client processes, ABI).
# Usage: bash scripts/host_sanitizers.sh [outdir]   (CPU only; run after the normal build)
set -u
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=${1:-$ROOT/gpurun_out}
mkdir -p "$OUT"
CUDA=${CUDA_HOME:-/usr/local/cuda}
KOBJ=$(ls "$ROOT"/build/svp/kernels_*.o)
TESTS="tests/test_plan.py tests/test_vp_control.py tests/test_ipc.py tests/test_abi.py tests/test_multiproc.py"
# TSan skips test_multiproc: torch's gloo process group reports races / mutex misuse on
# its own condition variables inside uninstrumented libtorch (no frame in libsvp); the
# library's threads (dispatcher, VP threads, IPC server) are covered by the other files
TSAN_TESTS="tests/test_plan.py tests/test_vp_control.py tests/test_ipc.py tests/test_abi.py"
SUPP=$ROOT/build/tsan.supp
mkdir -p "$ROOT/build"; printf 'called_from_lib:libtorch_cpu.so\nrace:libtorch_cpu.so\nmutex:libtorch_python.so\nmutex:libtorch_cpu.so\n' > "$SUPP"
for san in asan tsan; do
  B=$ROOT/build/$san; mkdir -p "$B"
  if [ $san = asan ]; then F="-fsanitize=address,undefined -fno-sanitize-recover=undefined"; RT=$(gcc -print-file-name=libasan.so)
  else F="-fsanitize=thread"; RT=$(gcc -print-file-name=libtsan.so); fi
  objs=""
  for src in "$ROOT"/paper_conf_dac_jungc15_b200/csrc/*.cpp; do
    o=$B/$(basename "$src").o
    g++ -O1 -g -fno-omit-frame-pointer -std=c++17 -fPIC $F -I"$CUDA/include" -I"$ROOT/include" -c "$src" -o "$o" || exit 1
    objs="$objs $o"
  done
  g++ -shared $F -o "$B/libsvp_$san.so" $objs $KOBJ -L"$CUDA/lib64" -lcudart_static -lpthread -ldl -lrt || exit 1
  ( cd "$ROOT" && SVP_LIB=$B/libsvp_$san.so LD_PRELOAD=$RT ASAN_OPTIONS=detect_leaks=0:abort_on_error=1 \
      UBSAN_OPTIONS=print_stacktrace=1:halt_on_error=1 TSAN_OPTIONS=halt_on_error=1:report_signal_unsafe=0:suppressions=$SUPP \
      timeout 900 python -m pytest $([ $san = tsan ] && echo $TSAN_TESTS || echo $TESTS) -q -m "not gpu" \
      -p no:cacheprovider > "$OUT/host_$san.log" 2>&1 )
  echo "$san rc=$?"; tail -2 "$OUT/host_$san.log"
  grep -c "ERROR: AddressSanitizer\|runtime error:\|WARNING: ThreadSanitizer" "$OUT/host_$san.log"
done
rm -rf "$ROOT/build/asan" "$ROOT/build/tsan"  # keep the gpurun snapshot small
