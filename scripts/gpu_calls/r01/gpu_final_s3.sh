# session-3 final pass: GPU tests, smoke, default bench, reference arm, IPC bench,
# ncu launch list + full capture of the bench's kernels
OUT=gpurun_out
bash scripts/gpu_full.sh
timeout 900 python tools/ipc_bench.py --calls 200 --out $OUT/ipc_bench200.json > $OUT/ipc_bench200.log 2>&1; echo "ipc rc=$?"
