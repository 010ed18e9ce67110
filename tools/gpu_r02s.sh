#!/bin/bash
O=gpurun_out/r02s; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
DGR_LIB=$PWD/gpurun_scratch_diag.so DGR_PROF_OUT=/tmp/tprof.bin timeout 600 python tools/tprof.py > $O/tprof.txt 2>&1; cat $O/tprof.txt
DGR_PARITY_COUNTS=$O/parity_counts.json timeout 2400 python -m pytest tests -q -m gpu -rf > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
grep -E "passed|failed|Error" $O/pytest_gpu.log | tail -12
