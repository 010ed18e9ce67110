#!/bin/bash
# r02 measurement pass: bench lines (ispd19 default incl. cpu_baseline + quality; c1e4; ispd18; ispd19 nets shuffled
# via ab_time), sweep, DGR* search, ncu launch list + full capture, sanitizers on the general path.
O=gpurun_out/r02m; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
timeout 900 python bench.py > $O/bench.log 2>&1; tail -1 $O/bench.log | cut -c1-300
for c in c1e4 ispd18 ispd19_c sweep4e6; do
  timeout 900 python bench.py --config $c --no-cpu-baseline --no-quality > $O/bench_$c.log 2>&1; tail -1 $O/bench_$c.log | cut -c1-200
done
timeout 900 python tools/sweep.py > $O/sweep.jsonl 2>$O/sweep.err; tail -4 $O/sweep.jsonl | cut -c1-200
timeout 1500 python tools/dgr_star.py 1-9 100 > $O/dgr_star.jsonl 2>$O/dgr_star.err; cat $O/dgr_star.jsonl | cut -c1-250
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 10 -c 60 --csv --log-file $O/launches.csv python tools/prof_run.py ispd19 8 > $O/ncu_launch.log 2>&1
for tool in memcheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/san_run.py tiny_m > $O/san_${tool}_tiny_m.log 2>&1
  echo "$tool tiny_m rc=$? $(tail -2 $O/san_${tool}_tiny_m.log | tr '\n' ' ')"
done
