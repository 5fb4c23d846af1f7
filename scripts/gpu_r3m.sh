# claim sizes now that the MTB side is faster: small-backlog threshold, tickets per small claim, lookahead
F=gpurun_out/r3m; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh sm1 "-DPAGODA_SMALL_MULT=1" cs2 "-DPAGODA_CLAIM_SMALL=2" lk2 "-DPAGODA_LOOKAHEAD=2" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 sm1 cs2 lk2; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs 2>/dev/null | tail -1 > $F/mb_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r3m/mm*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
