"""Workload definitions shared by tests/ and bench.py.

Holds only sizes and seeds (BASELINE.json ``configs``; XSBench defaults are
SURVEY.md App. A) -- none of the method's arithmetic.  Each side (oracle/ and the
CUDA library) implements the counter-based LCG that turns these seeds into inputs.
"""
from dataclasses import dataclass

GRID_SEED = 42          # XSBench grid seed [XSB] (reading R11)
LOOKUP_SEED = 1070      # XSBench STARTING_SEED [XSB]
HASH_BINS = 10000       # XSBench default hash bins [XSB]; BASELINE.json configs[4]

UNIONIZED, NUCLIDE, HASH = 0, 1, 2
GRID_NAMES = {UNIONIZED: "unionized", NUCLIDE: "nuclide", HASH: "hash"}


@dataclass(frozen=True)
class Workload:
    name: str
    n_nuclides: int
    n_gridpoints: int
    grid_type: int
    lookups: int          # strong scaling: the job's total; weak scaling: per rank
    note: str
    scaling: str = "strong"  # bench.py default (SURVEY.md §8e partitions a fixed total)

    @property
    def n_points(self) -> int:
        return self.n_nuclides * self.n_gridpoints


WORKLOADS = {
    # BASELINE.json configs[0]: the case the oracle finishes in seconds
    "tiny": Workload("tiny", 68, 1000, NUCLIDE, 100_000, "configs[0]"),
    # configs[1]: XSBench -s small (the paper's run), 1 GPU
    "small": Workload("small", 68, 11303, NUCLIDE, 17_000_000, "configs[1]"),
    # configs[2]: XSBench -s large, nuclide grid
    "large": Workload("large", 355, 11303, NUCLIDE, 17_000_000, "configs[2]"),
    # configs[3]: large, unionized (energy-index) grid
    "large-U": Workload("large-U", 355, 11303, UNIONIZED, 100_000_000, "configs[3]"),
    # configs[4]: XL, hash grid with 10,000 bins; 1e9 lookups over 8 GPUs
    # weak: every rank owns 125M lookups, so N = 8 is exactly the 1B-lookup configuration
    "XL": Workload("XL", 355, 238847, HASH, 1_000_000_000 // 8, "configs[4] (per-GPU share)", "weak"),
}

# Mean nuclides per lookup under pick_mat's effective distribution (SURVEY.md §8
# notation; [derived]); used only to state algorithmic bytes, never in results.
MEAN_NUCS = {68: 15.490, 355: 55.383}


# ---------------------------------------------------------------- bezier-surface (NEXT 4)
# The second u&u loop of the paper (Listing 2), run as a synthetic A/B.
# Table I runs bezier-surface with "-n 4096"; reading BZ3 takes
# that as a 4096 x 4096 output surface over a (NI+1) x (NJ+1) control net.
@dataclass(frozen=True)
class BezierWorkload:
    name: str
    ni: int
    nj: int
    res_i: int
    res_j: int
    note: str


BEZIER_SEED = 7
BEZIER_WORKLOADS = {
    "tiny": BezierWorkload("tiny", 5, 4, 61, 37, "oracle-sized, ragged against the 16 x 16 tiles"),
    "paper": BezierWorkload("paper", 5, 4, 4096, 4096, "-n 4096, NI=5, NJ=4 (reading BZ3)"),
    "deep": BezierWorkload("deep", 16, 16, 2048, 2048, "17 x 17 net: 16-trip Listing-2 loops"),
}


def bezier_control_net(ni: int, nj: int, seed: int = BEZIER_SEED, dtype="float64"):
    """Seeded control net P[(ni+1), (nj+1), 3]: a jittered lattice (x = ki, y = kj) with
    uniform heights in [0, 1) -- the shape of a terrain/patch input.  Input data only."""
    import numpy as np
    rng = np.random.default_rng(seed)
    P = np.zeros((ni + 1, nj + 1, 3), np.float64)
    P[..., 0] = np.arange(ni + 1)[:, None] + rng.uniform(-0.25, 0.25, (ni + 1, nj + 1))
    P[..., 1] = np.arange(nj + 1)[None, :] + rng.uniform(-0.25, 0.25, (ni + 1, nj + 1))
    P[..., 2] = rng.random((ni + 1, nj + 1))
    return P.astype(dtype)
