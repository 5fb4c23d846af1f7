# MM at 2 MTBs/SM with two scheduling groups and larger ingest stages; 3DES quad-sum variant
F=gpurun_out/r3a; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh qs "-DPAGODA_TDES_FULL_SUM=2" > $F/variants.log 2>&1
for i in 1 2; do
  for ak in 64 96 104; do
    timeout 200 python bench.py --workload mm --quick --no-configs --mtbs 2 --groups 2 --arena-kb $ak 2>/dev/null | tail -1 > $F/mm2g2a${ak}_0_$i.json
  done
  timeout 200 python bench.py --workload mm --quick --no-configs --mtbs 2 --arena-kb 104 2>/dev/null | tail -1 > $F/mm2g1a104_0_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_0_$i.json
  for v in 0 qs; do
    if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
    timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  done
  unset PAGODA_LIB
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r3a/mm*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
DRAIN=1 timeout 300 python scripts/probe_life.py mm nop > $F/life_drain.jsonl 2> $F/life.err; cat $F/life_drain.jsonl; tail -2 $F/life.err
