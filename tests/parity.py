"""GPU-vs-oracle comparison helpers (the acceptance rules of BASELINE.json's north_star)."""
import numpy as np

# fp32 edge values / probabilities: 1e-5 relative (north_star).
RTOL = 1e-5


def host_graph(g):
    """synth graph dict -> numpy arrays."""
    w = g["weights"]
    return (g["indptr"].cpu().numpy(), g["indices"].cpu().numpy(),
            None if w is None else w.cpu().numpy())


def compare_block(gpu, ref, where, float_keys=("val", "row_prob")):
    for k in ["col_map", "row_map", "indptr", "row_local", "eid"]:
        a, b = gpu[k], ref[k]
        assert a.shape == b.shape, f"{where}: {k} shape {a.shape} != {b.shape}"
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0]
            raise AssertionError(f"{where}: {k} differs at {bad[:5]} ({len(bad)} of {len(a)}): "
                                 f"gpu {a[bad[:5]]} ref {b[bad[:5]]}")
    for k in float_keys:
        a, b = gpu.get(k), ref.get(k)
        # an empty array and an absent (NULL) one are the same block: a
        # std::vector with no elements has no data pointer on the oracle side
        if a is not None and a.size == 0 and b is None:
            a = None
        if b is not None and b.size == 0 and a is None:
            b = None
        assert (a is None) == (b is None), f"{where}: {k} presence differs"
        if a is not None:
            np.testing.assert_allclose(a, b, rtol=RTOL, atol=0, err_msg=f"{where}: {k}")


def compare_all(gpu_blocks, ref_blocks, tag=""):
    assert len(gpu_blocks) == len(ref_blocks), f"{tag}: batch count"
    for b, (gl, rl) in enumerate(zip(gpu_blocks, ref_blocks)):
        assert len(gl) == len(rl)
        for l, (gb, rb) in enumerate(zip(gl, rl)):
            compare_block(gb, rb, f"{tag} batch {b} layer {l}")


def count_selection_mismatches(gpu_blocks, ref_blocks):
    """For weighted (A-Res) selections: number of blocks whose selected set differs."""
    bad = 0
    for gl, rl in zip(gpu_blocks, ref_blocks):
        for gb, rb in zip(gl, rl):
            if not np.array_equal(gb["eid"], rb["eid"]):
                bad += 1
    return bad
