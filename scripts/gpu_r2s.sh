# Round-2 session-2 baseline: HEAD's GPU suite + quick bench of the main workloads
F=gpurun_out/r2s; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $F/pytest_gpu.log 2>&1
for w in tdes mm mb mix nop; do for i in 1 2; do
  timeout 300 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json
done; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1
tail -3 $F/pytest_gpu.log; cat $F/ab.txt
