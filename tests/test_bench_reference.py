"""bench.py's reference arm (the driver contract's --impl reference, tier framing: the oracle as it
stands, on the host cores) runs on CPU and prints the contract's JSON line; the all-cores oracle
(net shards in threads, partial demand summed) reproduces the single-thread oracle's loss."""
import json
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_reference_arm_prints_the_contract_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny", "--steps", "3",
                        "--warmup", "3"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "impl", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in line, k
    assert line["impl"] == "reference" and line["value"] > 0 and line["steps"] == 3 and line["warmup"] == 3
    assert line["cpu_baseline"]["cores"] >= 1 and line["e2e"]["h2d_bytes_per_step"] == 0


def test_sharded_oracle_equals_the_single_thread_oracle():
    import bench
    import forestgen
    import oracle
    f = forestgen.generate("c1e4")
    o = oracle.Oracle(f)
    W = oracle.weights()
    so = bench.ShardedOracle(f, 3)
    for _ in range(3):
        ref = o.step(1, 1.0, 0.3, W)
        got = so.step(1.0, 0.3)
        np.testing.assert_allclose(got, ref, rtol=1e-9)
    so.close()
