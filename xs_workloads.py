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
    lookups: int          # per GPU at N=1 (bench weak-scales this per rank)
    note: str

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
    "XL": Workload("XL", 355, 238847, HASH, 1_000_000_000 // 8, "configs[4] (per-GPU share)"),
}

# Mean nuclides per lookup under pick_mat's effective distribution (SURVEY.md §8
# notation; [derived]); used only to state algorithmic bytes, never in results.
MEAN_NUCS = {68: 15.490, 355: 55.383}
