# 8 MTBs/SM with the copy-engine ingest: occupancy diagnostics, CE tests, MM A/B
F=gpurun_out/r3f; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_ce_ingest.py -q -x > $F/pytest_ce.log 2>&1; tail -3 $F/pytest_ce.log
for ak in 20 16 12; do
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb $ak > $F/mm8a${ak}_dbg.txt 2>&1; grep -v "^ " $F/mm8a${ak}_dbg.txt | tail -3
done
for i in 1 2; do
  for ak in 16 12; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb $ak 2>/dev/null | tail -1 > $F/mm8a${ak}_ce1_$i.json
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb $ak --prespawn 2>/dev/null | tail -1 > $F/mm8a${ak}pre_ce1_$i.json
  done
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 2>/dev/null | tail -1 > $F/mm_ce1_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --producers 2 2>/dev/null | tail -1 > $F/mmp2_ce1_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --ce 1 2>/dev/null | tail -1 > $F/mb_ce1_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --ce 0 2>/dev/null | tail -1 > $F/mb_ce0_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r3f/mm*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
