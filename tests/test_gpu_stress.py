"""Protocol-stress tier (the single-kernel soft synchronisation must be
correct and deadlock-free under any CTA -> SM assignment and any relative speed of the CTAs).

* co-resident: a kernel holding all but a few SMs (sat_debug_occupy) runs while the SAT launches on
  another stream, so the SAT's persistent CTAs start over tens of milliseconds and the first few do all
  the work -- every element still equal to the oracle;
* jitter + watchdog: the parity worker (tests/stress_worker.py) against libsat_stress.so, built with
  -DSAT_JITTER=1 (random sleeps before every status-word publication) and -DSAT_WATCHDOG=1 (spins trap
  after 10 s instead of hanging), in a subprocess.
Needs a B200."""
import os
import subprocess
import sys
from pathlib import Path

import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = Path(__file__).resolve().parent.parent


@pytest.fixture(scope="module")
def sat():
    import paper_conf_ipps_emotofthni18_b200 as sat

    sat.set_tuning(-1, 0, 0)
    sat.set_max_ctas(0)
    yield sat
    sat.set_tuning(-1, 0, 0)


@pytest.mark.parametrize("rows,cols,free", [(1000, 1300, 4), (4096, 4096, 2), (6000, 6000, 3), (6000, 6000, 1)])
def test_sat_while_other_kernel_holds_most_sms(sat, rows, cols, free):
    dev = torch.device("cuda", 0)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    a = satgen.gen_host(rows, cols, seed=4242 + free, dist="u32")
    x = torch.from_numpy(a).to(dev)
    hog, work = torch.cuda.Stream(), torch.cuda.Stream()
    with torch.cuda.stream(work):
        sat.sat(x, stream=work)  # workspace of `work` grown before the occupied launch
    torch.cuda.synchronize()
    sat.debug_occupy(sms - free, 30_000_000, 200 * 1024, stream=hog)  # 30 ms on all but `free` SMs
    with torch.cuda.stream(work):
        out = sat.sat(x, stream=work)
    torch.cuda.synchronize()
    assert (out.cpu().numpy() == oracle.sat_i32(a)).all()


def test_chained_strips_while_other_kernel_holds_most_sms(sat):
    dev = torch.device("cuda", 0)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    rows, cols, n = 2000, 2600, 3
    a = satgen.gen_host(rows, cols, seed=4300, dist="u32")
    chains = sat.Chain.local(n, cols)
    try:
        parts = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + h])).to(dev)
                 for r0, h in (sat.strip_bounds(rows, n, r) for r in range(n))]
        streams = [torch.cuda.Stream() for _ in range(n)]
        hog = torch.cuda.Stream()
        for r in range(n):  # chain slot buffers grown before the occupied launch
            sat.sat_chained(parts[r], chain=chains[r], stream=streams[r])
        torch.cuda.synchronize()
        sat.debug_occupy(sms - 3, 30_000_000, 200 * 1024, stream=hog)
        outs = [sat.sat_chained(parts[r], chain=chains[r], stream=streams[r]) for r in range(n)]
        torch.cuda.synchronize()
        assert (torch.cat(outs).cpu().numpy() == oracle.sat_i32(a)).all()
    finally:
        for c in chains:
            c.close()


def test_occupy_argument_errors(sat):
    with pytest.raises(sat.SatError):
        sat.debug_occupy(0, 1000)
    with pytest.raises(sat.SatError):
        sat.debug_occupy(1, 1000, 300 * 1024)


def test_parity_under_jitter_and_watchdog():
    lib = ROOT / "paper_conf_ipps_emotofthni18_b200" / "libsat_stress.so"
    if not lib.exists():
        pytest.skip("libsat_stress.so not built (python build_native.py --stress)")
    env = dict(os.environ, SAT_LIB=str(lib))
    r = subprocess.run([sys.executable, str(ROOT / "tests" / "stress_worker.py"), "--reps", "3"], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "stress worker ok" in r.stdout
