# A/B: free-before-post (+CTA fences); MB at 1 MTB/SM with spread delays; a fresh full headline line.
O=gpurun_out/ab21; mkdir -p $O
VARS="0 fe fecta" AB=ab21 bash scripts/gpu_ab.sh
for ns in 6000 24000; do for m in 1 2; do for i in 1 2; do
  PAGODA_SPREAD_NS=$ns timeout 300 python bench.py --quick --workload mb --mtbs $m --arena-kb 96 2>/dev/null | tail -1 > $O/mbcfg_m${m}_sp${ns}_$i.json
  python -c "import json;d=json.loads(open('$O/mbcfg_m${m}_sp${ns}_$i.json').read().strip().splitlines()[-1]);print('mb m$m sp$ns', round(d['value']/1e6,2))"
done; done; done
timeout 900 python bench.py > $O/bench_tdes.json 2> $O/bench_tdes.err
python -c "import json;d=json.loads(open('$O/bench_tdes.json').read().strip().splitlines()[-1]);print('tdes', round(d['value']/1e6,2), d['latency']['loaded_us'], d['e2e']['value']/1e6, d['roofline']['frac'], d['clocks'])"
