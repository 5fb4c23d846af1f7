# fast contiguous shape validation (a SIMD scan instead of 5 compares per row) + parallel validation in MT spawns
F=gpurun_out/r3p; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_gpu_ce_ingest.py tests/test_cpp_api.py -q -x > $F/pytest.log 2>&1; tail -2 $F/pytest.log
for i in 1 2; do
  for w in tdes mm mb mix; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json; done
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
