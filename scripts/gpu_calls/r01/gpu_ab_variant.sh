# A/B of a tables.h constant: variant tree in /tmp/variant (sed expression $1), 3 alternating bench runs each
OUT=$PWD/gpurun_out; ROOTD=$PWD
rm -rf /tmp/variant && mkdir -p /tmp/variant && tar --exclude=./gpurun_out --exclude=./build -cf - . | tar -C /tmp/variant -xf -
sed -i "$1" /tmp/variant/paper_conf_dac_jungc15_b200/csrc/tables.h
grep -n "kBsVec =\|kVecaddVec =\|kHistVec =" /tmp/variant/paper_conf_dac_jungc15_b200/csrc/tables.h
(cd /tmp/variant && python -c "from paper_conf_dac_jungc15_b200 import _build; _build.build(force=True)") || echo "variant build failed"
for i in 1 2 3; do
  (cd $ROOTD && timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/ab_base_$i.log 2>&1)
  (cd /tmp/variant && timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/ab_var_$i.log 2>&1)
done
for f in $OUT/ab_base_*.log $OUT/ab_var_*.log; do tail -1 $f | python -c "import json,sys; d=json.loads(sys.stdin.read()); pk=d['per_kernel']; print('$(basename $f)', round(d['value']), round(d['ms_per_step'],3), {k: round(v['avg_launch_ms'],3) for k,v in pk.items()}, d['clocks']['sm_mhz'])"; done
