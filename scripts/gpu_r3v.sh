# MB claim caps with two scheduling groups per MTB (two holders)
F=gpurun_out/r3v; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  timeout 200 python bench.py --workload mb --quick --no-configs 2>/dev/null | tail -1 > $F/mb_m2g1_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --groups 2 --max-tasks 1 2>/dev/null | tail -1 > $F/mb_m1g2_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --groups 2 --max-tasks 2 2>/dev/null | tail -1 > $F/mb_m2g2_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --max-tasks 2 --producers 2 2>/dev/null | tail -1 > $F/mb_m2p2_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --ce 1 --max-tasks 2 --arena-kb 16 2>/dev/null | tail -1 > $F/mb_m2ce_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
