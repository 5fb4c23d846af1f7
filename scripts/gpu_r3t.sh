# shape-cache validation; C5 (1M mixed rows) with 1-8 producers (validation and spawning in parallel)
F=gpurun_out/r3t; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py -q -x -k "valid or producer or shapes or nop_many" > $F/pytest.log 2>&1; tail -2 $F/pytest.log
for i in 1 2; do
  for pr in 1 2 4 8; do timeout 300 python bench.py --workload c5 --quick --no-configs --steps 3 --warmup 1 --producers $pr 2>/dev/null | tail -1 > $F/c5_p${pr}_$i.json; done
  for w in tdes mm; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json; done
  timeout 200 python bench.py --workload mix --quick --no-configs --producers 4 2>/dev/null | tail -1 > $F/mix_p4_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_p2_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
