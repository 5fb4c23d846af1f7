timeout 600 python -m pytest tests/test_gpu_runtime.py -q -x -k "four or init_info" 2>&1 | tail -3
for r in 1 2; do
  line="r$r"
  for cfg in "mm|" "mm|--mtbs 4 --arena-kb 48" "nop|" "nop|--mtbs 4 --arena-kb 48" "mix|" "mix|--mtbs 4 --arena-kb 48" "mix|--mtbs 2 --arena-kb 96" "mb|" "mb|--mtbs 4 --arena-kb 48"; do
    w=${cfg%%|*}; extra=${cfg#*|}
    timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive --steps 5 $extra 2>/dev/null | tail -1 > gpurun_out/ab11.json
    line="$line $w[$extra]=$(python -c "import json;d=json.load(open('gpurun_out/ab11.json'));print(round(d['value']/1e6,2))" 2>/dev/null)"
  done
  echo $line
done
