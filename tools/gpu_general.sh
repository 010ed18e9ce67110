#!/bin/bash
O=gpurun_out/r02_gen; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for c in ispd18 ispd18_m c1e4 c1e4_m; do python tools/ab_time.py $c 200 3; done 2>&1 | grep -v Warning | tee $O/ab.jsonl | cut -c1-330
timeout 900 python bench.py --config ispd18_m --no-cpu-baseline --no-quality > $O/bench_ispd18_m.log 2>&1; tail -1 $O/bench_ispd18_m.log | cut -c1-300
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 10 -c 30 --csv --log-file $O/launches.csv python tools/prof_run.py ispd18_m 5 > $O/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf_m python tools/prof_run.py ispd18_m 3 > $O/ncu_full.log 2>&1
ls $O
