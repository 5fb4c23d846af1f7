F=gpurun_out/r3u; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  for w in tdes mm mb mix; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json; done
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 3 --warmup 1 2>/dev/null | tail -1 > $F/c5_0_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
