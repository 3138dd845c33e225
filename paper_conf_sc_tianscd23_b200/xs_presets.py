"""The five BASELINE.json workloads (no library import needed).

Seeds follow DESIGN.md R1: grid 42, concentrations 1070^2, lookups 1070 (the
XSBench values; with them the oracle reproduces XSBench's published event
checksums 945990 / 952131 for small / large).
"""
# BASELINE.json configs; seeds per DESIGN.md R1 (grid 42, conc 1070^2, lookups 1070)
PRESETS = {
    "tiny": dict(n_isotopes=12, n_gridpoints=1000, material_rule=1, lookups=100_000,
                 grid_type="unionized"),
    "small": dict(n_isotopes=68, n_gridpoints=11303, material_rule=0, lookups=17_000_000,
                  grid_type="unionized"),
    "large": dict(n_isotopes=355, n_gridpoints=11303, material_rule=0, lookups=17_000_000,
                  grid_type="unionized"),
    "large-hash": dict(n_isotopes=355, n_gridpoints=11303, material_rule=0, lookups=17_000_000,
                       grid_type="hash", hash_bins=8192, sort=True),
    "xl": dict(n_isotopes=355, n_gridpoints=238847, material_rule=0, lookups=170_000_000,
               grid_type="unionized"),
}
GRID_SEED, CONC_SEED, LOOKUP_SEED = 42, 1070 * 1070, 1070


