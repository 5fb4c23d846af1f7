# copy-engine ingest, bounded copies in flight: tests, then A/B (doorbell vs CE, 4 and 8 MTBs/SM)
F=gpurun_out/r3e; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_ce_ingest.py -q -x > $F/pytest_ce.log 2>&1
PAGODA_TEST_FLAGS=0x40 timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py -q > $F/pytest_rt_ce.log 2>&1
tail -3 $F/pytest_ce.log; tail -5 $F/pytest_rt_ce.log
timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb 20 > $F/mm8_dbg.txt 2>&1; tail -5 $F/mm8_dbg.txt
for i in 1 2; do
  for ce in 0 1; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce $ce 2>/dev/null | tail -1 > $F/mm_ce$ce\_$i.json
    timeout 200 python bench.py --workload mm --quick --no-configs --ce $ce --prespawn 2>/dev/null | tail -1 > $F/mmpre_ce$ce\_$i.json
    timeout 200 python bench.py --workload nop --quick --no-configs --ce $ce 2>/dev/null | tail -1 > $F/nop_ce$ce\_$i.json
    timeout 200 python bench.py --workload tdes --quick --no-configs --ce $ce 2>/dev/null | tail -1 > $F/tdes_ce$ce\_$i.json
  done
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb 20 2>/dev/null | tail -1 > $F/mm8_ce1_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --mtbs 8 --arena-kb 20 --prespawn 2>/dev/null | tail -1 > $F/mm8pre_ce1_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r3e/mm*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
