# MB: more schedulers per SM with a claim cap of 1 (now that a cap of 1 drains correctly)
F=gpurun_out/r4b; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  timeout 200 python bench.py --workload mb --quick --no-configs 2>/dev/null | tail -1 > $F/mb_preset_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs 2 --arena-kb 40 --max-tasks 1 2>/dev/null | tail -1 > $F/mb_m2c1_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs 2 --arena-kb 40 --max-tasks 2 2>/dev/null | tail -1 > $F/mb_m2c2_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs 4 --arena-kb 16 --ce 1 --max-tasks 1 2>/dev/null | tail -1 > $F/mb_m4c1ce_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs 1 --max-tasks 3 --groups 2 2>/dev/null | tail -1 > $F/mb_m1c3g2_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
