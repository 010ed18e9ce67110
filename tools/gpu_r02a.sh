#!/bin/bash
# r02 first pass: build + smoke, full gpu tests (data-gathering K_PROBE), sanitizers, bench line.
O=gpurun_out/r02a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
DGR_K_PROBE=1e9 DGR_PARITY_COUNTS=$O/parity_counts.json timeout 1800 python -m pytest tests -q -m gpu -rf > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -60 $O/pytest_gpu.log
for cfg in tiny c1e4; do
  for tool in memcheck racecheck synccheck initcheck; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/san_run.py $cfg > $O/san_${tool}_${cfg}.log 2>&1
    echo "$tool $cfg rc=$? $(tail -2 $O/san_${tool}_${cfg}.log | tr '\n' ' ')"
  done
done
DGR_ALL_SLOW=1 timeout 900 compute-sanitizer --tool memcheck python tools/san_run.py c1e4 > $O/san_memcheck_c1e4_slow.log 2>&1
echo "memcheck slow rc=$? $(tail -2 $O/san_memcheck_c1e4_slow.log | tr '\n' ' ')"
DGR_ALL_SLOW=1 timeout 900 compute-sanitizer --tool racecheck python tools/san_run.py c1e4 > $O/san_racecheck_c1e4_slow.log 2>&1
echo "racecheck slow rc=$? $(tail -2 $O/san_racecheck_c1e4_slow.log | tr '\n' ' ')"
timeout 900 python bench.py > $O/bench.log 2>&1; tail -1 $O/bench.log | cut -c1-600
