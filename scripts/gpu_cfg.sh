# Context-configuration sweep (MTBs per SM, spread delay) on the bench workloads (quick lines).
O=gpurun_out/cfg; mkdir -p $O
run() { tag=$1; shift; for i in 1 2; do timeout 300 python bench.py --quick "$@" 2>/dev/null | tail -1 > $O/${tag}_$i.json; done
  python - $O/${tag}_1.json $O/${tag}_2.json <<'P'
import json, sys
v = []
for f in sys.argv[1:]:
    try: v.append(round(json.loads(open(f).read().strip().splitlines()[-1])["value"] / 1e6, 2))
    except Exception: v.append(None)
print(sys.argv[1].split("/")[-1][:-7], v)
P
}
run mm_m4 --workload mm
run mm_m2 --workload mm --mtbs 2 --arena-kb 96
run mm_m1 --workload mm --mtbs 1 --arena-kb 200
run nop_m2 --workload nop
run nop_m4 --workload nop --mtbs 4 --arena-kb 48
run mix_m1 --workload mix
run mix_m2 --workload mix --mtbs 2 --arena-kb 96
run c5_m1 --workload c5
run c5_m2 --workload c5 --mtbs 2 --arena-kb 96
for ns in 3000 6000 12000 24000; do PAGODA_SPREAD_NS=$ns run mb_sp$ns --workload mb; done
PAGODA_SPREAD_NS=6000 run mb_m1_sp6000 --workload mb --mtbs 1 --arena-kb 96
for i in 1 2; do timeout 600 python bench.py --no-naive --no-cpu > $O/tdes_full_$i.json 2>/dev/null
  python -c "import json;d=json.loads(open('$O/tdes_full_$i.json').read().strip().splitlines()[-1]);print('tdes', round(d['value']/1e6,2), d['latency']['loaded_us'], d['e2e']['value']/1e6)"; done
