# preset candidates: MM (CE, arena, producers), 3DES arena, MB arena, MM variants
F=gpurun_out/r3j; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do
  for ak in 16 20 24; do for pr in 2 3; do
    timeout 200 python bench.py --workload mm --quick --no-configs --ce 1 --arena-kb $ak --producers $pr 2>/dev/null | tail -1 > $F/mm_a${ak}p${pr}_$i.json
  done; done
  timeout 200 python bench.py --workload mm_tc --quick --no-configs --ce 1 --arena-kb 24 --producers 2 2>/dev/null | tail -1 > $F/mmtc_a24p2_$i.json
  timeout 200 python bench.py --workload mm_tc --quick --no-configs 2>/dev/null | tail -1 > $F/mmtc_preset_$i.json
  timeout 200 python bench.py --workload mm_noshm --quick --no-configs --ce 1 --arena-kb 8 --producers 2 2>/dev/null | tail -1 > $F/mmnoshm_a8p2_$i.json
  timeout 200 python bench.py --workload mm_noshm --quick --no-configs 2>/dev/null | tail -1 > $F/mmnoshm_preset_$i.json
  for ak in 8 4; do timeout 200 python bench.py --workload tdes --quick --no-configs --arena-kb $ak 2>/dev/null | tail -1 > $F/tdes_a${ak}_$i.json; done
  timeout 200 python bench.py --workload tdes_var --quick --no-configs --arena-kb 8 2>/dev/null | tail -1 > $F/tdesvar_a8_$i.json
  timeout 200 python bench.py --workload tdes_var --quick --no-configs 2>/dev/null | tail -1 > $F/tdesvar_preset_$i.json
  for ak in 8 16; do timeout 200 python bench.py --workload mb --quick --no-configs --arena-kb $ak 2>/dev/null | tail -1 > $F/mb_a${ak}_$i.json; done
  timeout 200 python bench.py --workload nop --quick --no-configs --ce 1 --arena-kb 16 2>/dev/null | tail -1 > $F/nop_ce16_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
