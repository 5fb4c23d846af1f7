# CE ingest with events (one memop per copy, 3 in flight): tests; MM CE + small arenas; 3DES / C5 / mix arena sweeps (L1 for spills)
F=gpurun_out/r3i; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_ce_ingest.py -q -x > $F/pytest_ce.log 2>&1; tail -2 $F/pytest_ce.log
PAGODA_TEST_FLAGS=0x40 timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py -q > $F/pytest_rt_ce.log 2>&1; tail -2 $F/pytest_rt_ce.log
for i in 1 2; do
  for ak in 24 16; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb $ak 2>/dev/null | tail -1 > $F/mmce_a${ak}_$i.json
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb $ak --producers 2 2>/dev/null | tail -1 > $F/mmcep2_a${ak}_$i.json
  done
  timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb 16 --prespawn 2>/dev/null | tail -1 > $F/mmcepre_a16_$i.json
  for ak in 40 24 16 8; do
    timeout 200 python bench.py --workload tdes --quick --no-configs --arena-kb $ak 2>/dev/null | tail -1 > $F/tdes_a${ak}_$i.json
  done
  timeout 200 python bench.py --workload tdes --quick --no-configs --arena-kb 8 --ce 1 2>/dev/null | tail -1 > $F/tdesce_a8_$i.json
  timeout 200 python bench.py --workload c5 --quick --no-configs --steps 2 --warmup 1 2>/dev/null | tail -1 > $F/c5_a144_$i.json
  timeout 200 python bench.py --workload c5 --quick --no-configs --steps 2 --warmup 1 --arena-kb 100 2>/dev/null | tail -1 > $F/c5_a100_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs --arena-kb 160 2>/dev/null | tail -1 > $F/mix_a160_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_a200_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --arena-kb 32 2>/dev/null | tail -1 > $F/mb_a32_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
