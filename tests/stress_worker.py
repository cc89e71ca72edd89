"""Protocol-stress worker (PAPER.md:21 -- correct under any CTA -> SM assignment and
any relative CTA speed).  Runs every shipped kernel family of whatever libsat SAT_LIB names (the product,
or libsat_stress.so built with -DSAT_JITTER=1 -DSAT_WATCHDOG=1) on small ragged shapes, forced onto each
variant, several times, and compares every element with the CPU oracle.  Run as a script (by
tests/test_gpu_stress.py, or under compute-sanitizer by tools/sanitize.sh); exit status 0 = all equal.

    python tests/stress_worker.py [--reps N] [--quick]
"""
from __future__ import annotations

import argparse
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402


VERBOSE = False


def note(what: str) -> None:
    if VERBOSE:
        print("case:", what, flush=True)


def check(got: np.ndarray, a: np.ndarray, dist: str, what: str) -> None:
    if dist in ("u32", "u8"):
        want = oracle.sat_u32(a.astype(np.uint32)) if dist == "u8" else oracle.sat_i32(a)
        got = got.view(np.uint32) if dist == "u8" else got
        if not (got == want).all():
            bad = np.argwhere(got != want)
            raise AssertionError(f"{what}: {len(bad)} mismatches, first at {bad[0].tolist()}")
    else:
        b, ab = oracle.sat_f32(a)
        if not (np.abs(got.astype(np.float64) - b) <= oracle.f32_tolerance(ab, *a.shape)).all():
            raise AssertionError(f"{what}: fp32 outside the R10 tolerance")


def main() -> int:
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--quick", action="store_true", help="one shape per variant (compute-sanitizer runs)")
    ap.add_argument("--verbose", action="store_true", help="print every case before it runs")
    args = ap.parse_args()
    global VERBOSE
    VERBOSE = args.verbose
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    shapes = [(300, 517), (1000, 1300), (777, 3001), (2048, 2048)]
    if args.quick:
        shapes = [(300, 1100)]
    # (variant, dists): 0 classic 64x128, 1 TMEM-parked 128x128, 3 TMEM-parked flat 64x256
    variants = [(0, ("u32", "fsym")), (1, ("u32", "fsym")), (3, ("u32", "fsym"))]
    n = 0
    try:
        for rep in range(args.reps):
            for vi, dists in variants:
                sat.set_tuning(vi, 0, 0)
                for rows, cols in shapes:
                    for dist in dists:
                        a = satgen.gen_host(rows, cols, seed=1000 + rows + rep, dist=dist)
                        note(f"variant {vi} {rows}x{cols} {dist} rep {rep}")
                        got = sat.sat(torch.from_numpy(a).to(dev)).cpu().numpy()
                        check(got, a, dist, f"variant {vi} {rows}x{cols} {dist} rep {rep}")
                        n += 1
                # carry row (the sharded path's injection) on the same variant
                note(f"variant {vi} carry row rep {rep}")
                a = satgen.gen_host(700, 900, seed=77 + rep, dist="u32")
                top = 300
                carry = oracle.sat_i32(a)[top - 1]  # the SAT row above the strip (sat()'s carry argument)
                got = sat.sat(torch.from_numpy(np.ascontiguousarray(a[top:])).to(dev),
                              carry=torch.from_numpy(carry.copy()).to(dev)).cpu().numpy()
                want = oracle.sat_i32(a)[top:]
                if not (got == want).all():
                    raise AssertionError(f"variant {vi} carry row rep {rep}")
                n += 1
            sat.set_tuning(-1, 0, 0)
            # u8 integral images: 128 x 128 (variant 2) and flat 64 x 256 (variant 5) kernels
            for uv in (2, 5):
                sat.set_tuning(uv, 0, 0)
                for rows, cols in shapes[:2]:
                    img = satgen.gen_host(rows, cols, seed=50 + rep, dist="u8").astype(np.uint8)
                    note(f"u8 variant {uv} {rows}x{cols} rep {rep}")
                    got = sat.sat_u8(torch.from_numpy(img).to(dev)).cpu().numpy()
                    check(got, img, "u8", f"u8 variant {uv} {rows}x{cols} rep {rep}")
                    n += 1
            sat.set_tuning(-1, 0, 0)
            # chained strips: 3 ranks, concurrent on their own streams (inbox pushes, polls, back-pressure)
            rows, cols, nr = 1500, 1300, 3
            note(f"chained strips rep {rep}")
            a = satgen.gen_host(rows, cols, seed=90 + rep, dist="u32")
            chains = sat.Chain.local(nr, cols)
            streams = [torch.cuda.Stream() for _ in range(nr)]
            sat.set_max_ctas(24)
            try:
                parts = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + h])).to(dev)
                         for r0, h in (sat.strip_bounds(rows, nr, r) for r in range(nr))]
                torch.cuda.synchronize()
                outs = []
                for _ in range(2):
                    outs.append([sat.sat_chained(parts[r], chain=chains[r], stream=streams[r]) for r in range(nr)])
                torch.cuda.synchronize()
                want = oracle.sat_i32(a)
                for k, o in enumerate(outs):
                    if not (torch.cat(o).cpu().numpy() == want).all():
                        raise AssertionError(f"chained strips call {k} rep {rep}")
                    n += 1
            finally:
                sat.set_max_ctas(0)
                for c in chains:
                    c.close()
    finally:
        sat.set_tuning(-1, 0, 0)
    torch.cuda.synchronize()
    print(f"stress worker ok: {n} cases, lib {sat._lib.LIB_PATH.name}")
    return 0


if __name__ == "__main__":
    sys.exit(main())
