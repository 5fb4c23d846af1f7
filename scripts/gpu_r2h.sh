F=gpurun_out/r2h; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
for m in 1 2; do for ew in 8 16 32; do for sp in 0 1; do
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs $m --exec-warps $ew --spread $sp 2>/dev/null | tail -1 > $F/mb_m${m}_e${ew}_s${sp}.json
  python -c "import json;d=json.loads(open('$F/mb_m${m}_e${ew}_s${sp}.json').read());print('mb m$m ew$ew sp$sp', round(d['value']/1e6,2))" >> $F/mb_sweep.txt 2>&1
done; done; done
tail -5 $F/pytest_gpu.log; cat $F/mb_sweep.txt
