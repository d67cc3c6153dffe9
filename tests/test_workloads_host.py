"""Host-side argument checks of the workload launch helpers (no GPU: they fail before any
device work)."""
import numpy as np
import pytest

from paper_conf_cgo_georgakoudispb25_b200 import workloads as W


def _tables(n_nuc, n_grid, n_mat):
    # shape-only stand-ins: the check runs before any array is touched
    e = np.zeros(1)
    return dict(egrid=e, recs=e, conc=e, cum=e, mat_nuc=e, mat_off=e, mat_cnt=e,
                n_nuc=n_nuc, n_grid=n_grid, n_mat=n_mat)


@pytest.mark.parametrize("n_nuc,n_grid,n_mat", [(355, 2 * 10 ** 6, 12), (68, 11303, 17),
                                                (64, 2 ** 20, 12)])
def test_xs_tables_beyond_the_kernel_index_bounds_are_rejected(n_nuc, n_grid, n_mat):
    """xs_lookup indexes recs with 32-bit flat offsets and shuffles a bracket's flat start
    row with its width in one word (n_nuc * n_grid < 2^26), and packs the material into
    perm's top 4 bits (n_mat <= 16)."""
    with pytest.raises(ValueError):
        W.xs_device_tables(_tables(n_nuc, n_grid, n_mat), device="cpu")


def test_xs_tables_at_the_configs_pass_the_check():
    d = W.xs_device_tables(_tables(68, 11303, 12), device="cpu")   # CFG 3
    assert d["n_nuc"] == 68 and d["gidx"] is None
    d = W.xs_device_tables(_tables(355, 11303, 12), device="cpu")  # NEXT-3 large table
    assert d["n_grid"] == 11303
    d = W.xs_device_tables(_tables(64, 2 ** 20 - 1, 12), device="cpu")   # just below 2^26
    assert d["n_nuc"] == 64


def test_adam_run_sfu_count_matches_the_kernel_source():
    """The SFU roofline of adam_run (bench.py, bench_suite.py) counts sqrt + rcp per
    element-step; the reciprocals of ADAM_RCP_SPLIT of a float4's 4 elements run on the FMA
    pipe instead (adam_step.cu).  Keep the constant in step with the kernel's defaults."""
    import re
    src = W.kernel_source("adam_run")
    fold = int(re.search(r"#define ADAM_FOLD (\d+)", src).group(1))
    m = re.search(r"#define ADAM_RCP_SPLIT \(ADAM_FOLD \? (\d+) : (\d+)\)", src)
    split = int(m.group(1) if fold else m.group(2))
    assert W.ADAM_RUN_SFU_PER_ELEMENT_STEP[1] == 2 - split / 4      # sqrt + rcp
    assert W.ADAM_RUN_SFU_PER_ELEMENT_STEP[0] == 1                  # one rsqrt
