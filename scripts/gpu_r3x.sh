F=gpurun_out/r3x; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_gpu_ce_ingest.py -q -x > $F/pytest.log 2>&1; tail -3 $F/pytest.log
for w in mb tdes; do timeout 150 python bench.py --workload $w --quick --no-configs --max-tasks 1 > $F/out_$w.txt 2>&1; echo "$w max_tasks 1 rc=$?"; done
for i in 1 2; do for w in tdes mm mb; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json; done; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
