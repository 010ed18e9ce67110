#!/bin/bash
O=gpurun_out/r02r; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1 || { tail -30 $O/build_smoke.log; exit 1; }
for r in 1 2; do
python tools/ab_time.py ispd19 200 3
python tools/ab_time.py ispd19+nshuf 200 3
done 2>&1 | grep -v Warning | tee $O/ab.jsonl
for i in 1 2 3; do timeout 600 python -m pytest tests/test_gpu_multiprocess.py -q -m gpu -x > $O/pytest_mp_$i.log 2>&1; tail -1 $O/pytest_mp_$i.log; done
cp paper_conf_dac_0159layhrr24_b200/csrc/dgr_kernels.cu $O/
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf_nshuf python tools/prof_run.py ispd19+nshuf 3 > $O/ncu_full_nshuf.log 2>&1
