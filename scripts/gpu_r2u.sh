# MTB concurrency (trace probe) + MB claim cap sweep (pagoda_config.max_tasks x spread)
F=gpurun_out/r2u; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 300 python scripts/probe_sched.py mm tdes nop > $F/probe_sched.jsonl 2> $F/probe_sched.err
for i in 1 2; do
  for mt in 0 2 3 4; do for sp in 1 0; do
    timeout 200 python bench.py --workload mb --quick --no-configs --max-tasks $mt --spread $sp 2>/dev/null | tail -1 > $F/mb_m${mt}s${sp}_$i.json
  done; done
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt; cat $F/probe_sched.jsonl; tail -3 $F/probe_sched.err
