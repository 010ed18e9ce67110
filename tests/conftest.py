import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (runs the sm_100a kernels through the C-ABI)")
    config.addinivalue_line("markers", "slow: larger CPU cases")


@pytest.fixture(scope="session")
def tiny():
    import forestgen
    return forestgen.generate("tiny")


@pytest.fixture(scope="session")
def c1e4():
    import forestgen
    return forestgen.generate("c1e4")


@pytest.fixture(scope="session", params=["tiny", "tiny_c", "tiny_m"])
def tinyx(request):
    """tiny, tiny with C-shape detours (row f4, reading Q14b), and tiny with monotone staircases and
    groups of more than 32 candidates (row f4', reading Q14c)"""
    import forestgen
    return forestgen.generate(request.param)


def pytest_terminal_summary(terminalreporter, exitstatus, config):
    """Clause counts of the float parity contract (tests/test_gpu_parity.py compare_state): how many
    elements passed strictly (<= 1e-4), through the fp32-probe clause, or as exempt first-step
    coordinates, per test and field.  Also written to $DGR_PARITY_COUNTS (default
    gpurun_out/parity_counts.json)."""
    import json
    mod = sys.modules.get("tests.test_gpu_parity")
    counts = getattr(mod, "PARITY_COUNTS", None) if mod else None
    if not counts:
        return
    tr = terminalreporter
    tr.write_sep("-", "float parity clause counts (strict / fp32-probe / exempt / chaotic / bad of n; "
                      "K_PROBE=%g KAPPA=%g)" % (mod.K_PROBE, mod.KAPPA))
    for what, fields in counts.items():
        for nm, c in fields.items():
            if "strict" in c and "n" in c:
                tr.write_line(f"{what:34s} {nm:7s} n={c['n']:>9d} strict={c['strict']:>9d} probe={c.get('probe', 0):>6d} "
                              f"exempt={c.get('exempt', c.get('tie', 0)):>6d} chaotic={c.get('chaotic', 0):>4d} "
                              f"bad={c.get('bad', 0):>3d} max_err={c.get('max_err', c.get('max_abs_tie', 0)):.2e} "
                              f"max_ratio={c.get('max_probe_ratio', 0):.2f} fp32>tol={c.get('fp32_beyond_tol', 0)} "
                              f"fp32_max={c.get('fp32_max_err', 0):.2e}")
            else:
                tr.write_line(f"{what:34s} {nm:7s} " + " ".join(f"{k}={v}" for k, v in c.items()))
    out = os.environ.get("DGR_PARITY_COUNTS", os.path.join(ROOT, "gpurun_out", "parity_counts.json"))
    try:
        os.makedirs(os.path.dirname(out), exist_ok=True)
        with open(out, "w") as fh:
            json.dump({"K_PROBE": mod.K_PROBE, "KAPPA": mod.KAPPA, "CHAOS_DEMAND": mod.CHAOS_DEMAND,
                       "counts": counts}, fh, indent=1)
    except OSError:
        pass
