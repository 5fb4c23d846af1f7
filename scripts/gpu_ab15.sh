# A/B: host producer threads (1..4) per workload, and MB at 1 MTB/SM (two-pixel body) vs 2.
mkdir -p gpurun_out/ab15
O=gpurun_out/ab15
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "mandelbrot or fusion or naive" > $O/t_mb.txt 2>&1
for w in nop mm tdes mix; do for pr in 1 2 3 4; do for i in 1 2; do
  timeout 300 python bench.py --workload $w --quick --producers $pr 2>/dev/null | tail -1 > $O/${w}_p${pr}_$i.json
done; done; done
for m in 1 2; do for pr in 1 2; do for i in 1 2; do
  timeout 300 python bench.py --workload mb --quick --mtbs $m --producers $pr 2>/dev/null | tail -1 > $O/mb_m${m}p${pr}_$i.json
done; done; done
timeout 300 python bench.py --workload mb --mtbs 1 --no-cpu > $O/mb_full_m1.json 2>$O/mb_full_m1.err
python - <<'P'
import glob, json, os
for f in sorted(glob.glob("gpurun_out/ab15/*_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1]); print(os.path.basename(f), round(d["value"]/1e6, 2))
    except Exception as e: print(f, "ERR", e)
P
tail -3 $O/t_mb.txt
