#!/bin/bash
O=gpurun_out/r02o; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
for r in 1 2; do
python tools/ab_time.py ispd19 200 3
python tools/ab_time.py ispd19+nshuf 200 3
DGR_LIB=$PWD/gpurun_scratch_head.so python tools/ab_time.py ispd19 200 3
done 2>&1 | grep -v Warning | tee $O/ab.jsonl
DGR_PARITY_COUNTS=$O/parity_counts.json timeout 2400 python -m pytest tests -q -m gpu -rf -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
grep -E "passed|failed|Error" $O/pytest_gpu.log | tail -12
cp paper_conf_dac_0159layhrr24_b200/csrc/dgr_kernels.cu $O/
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu_full.log 2>&1
