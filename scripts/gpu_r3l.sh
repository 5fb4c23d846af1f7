# idle back-off cap of schedulers / I/O warps (PAGODA_IDLE_NS): isolated latency and throughput
F=gpurun_out/r3l; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh i512 "-DPAGODA_IDLE_NS=512" i256 "-DPAGODA_IDLE_NS=256" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 i512 i256; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python bench.py --no-configs --no-e2e --no-cpu 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r3l/tdes_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), d["latency"]["isolated_nop128_us"], round(d["latency"]["isolated_nop128_over_floor"],3))
    except Exception as e: print(f, e)
PY
