# NEXT f4: parity of hetero / graph, then A/B of the four option combinations on cfg5
OUT=gpurun_out
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_f4.py -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_f4.log 2>&1; echo "pytest f4 rc=$?"; grep -E "passed|failed|FAILED|Error" $OUT/pytest_f4.log | tail -12
for hg in "0 0" "1 0" "0 1" "1 1"; do
  set -- $hg
  timeout 600 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-alt --hetero $1 --graph $2 > $OUT/bench_h$1_g$2.log 2>&1; echo "hetero=$1 graph=$2 rc=$?"
done
