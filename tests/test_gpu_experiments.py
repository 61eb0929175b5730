"""GPU checks of the paper's other evaluation modes (PAPER.md S6), run through
paper_conf_ppopp_mccoyp24_b200.experiments on the C-ABI bulk calls.

* Utilization (E8): successes until the first NULL obey the
  closed forms of the paper's geometry (the same bounds tests/test_oracle_alloc.py
  pins O2 to), every returned pointer is stamp-verified and accounted, and
  freeing everything after the out-of-memory state drains to the pristine image.
* Fragmentation (E7): the address range of 2^20 live slices is at
  least the packed size and the heap stays consistent.
* Warm-up (E6) and variance (E5): rounds without a reset stay
  correct; the timing fields are well formed.
* Init (E1): init/destroy cycles leave a pristine allocator.
"""
import numpy as np
import pytest
import torch

import workload_gen as wg
from helpers import SEG, class_size, diff_images, pristine_image

pytestmark = pytest.mark.gpu


@pytest.fixture()
def G():
    import paper_conf_ppopp_mccoyp24_b200 as G
    yield G
    if G.gallatin_is_initialized():
        G.gallatin_destroy()


@pytest.fixture()
def X():
    from paper_conf_ppopp_mccoyp24_b200 import experiments
    return experiments


def _pristine(G, nseg):
    G.gallatin_drain()
    img = G.gallatin_snapshot()
    msg = diff_images(img, pristine_image(nseg, int(img[4])))
    assert not msg, msg


@pytest.mark.parametrize("size", [4, 16, 64, 512, 4096, 8192, 1 << 20, 1 << 24, 3 << 24])
def test_utilization_closed_form(cuda_ok, G, X, size):
    nseg = 16
    G.gallatin_init(nseg * SEG)
    r = X.utilization(size)
    succ = r["successes"]
    st = G.gallatin_stats()
    if size <= 4096:
        c = max(0, (size - 1).bit_length() - 4)
        total = nseg * (256 >> c) * 4096
        assert total - st["nslot"][c] * 4096 <= succ <= total, (succ, total)
    elif size < SEG:
        t = max(0, (size - 1).bit_length() - 16)
        assert succ == nseg * (256 >> t)
    else:
        assert succ == nseg // -(-size // SEG)
    assert st["errors"] == 0
    ptrs = torch.cat(r["ptrs"])
    live = ptrs[ptrs != 0].contiguous()
    sizes = torch.full_like(live, size)
    G.gallatin_stamp(live, sizes)
    assert G.gallatin_verify(live, sizes) == 0
    usum, ubad = G.gallatin_usable(live, sizes)
    assert ubad == 0 and usum == succ * class_size(size)
    G.gallatin_free(live)
    _pristine(G, nseg)


@pytest.mark.parametrize("size", [16, 256, 4096])
def test_fragmentation_range(cuda_ok, G, X, size):
    """E7 with the default knobs: every request granted, the range at least
    the bytes requested and inside the heap, accounting exact, pristine after."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    r = X.fragmentation(size, 1 << 20)
    assert r["nulls"] == 0
    assert r["range_bytes"] >= ((1 << 20) - 1) * size
    assert r["range_bytes"] < nseg * SEG
    usum, ubad = G.gallatin_usable(r["ptrs"], r["sizes"])
    assert ubad == 0 and usum == (1 << 20) * size
    G.gallatin_free(r["ptrs"])
    _pristine(G, nseg)


def test_fragmentation_paper_policy_front_first(cuda_ok, G, X):
    """E7 under the paper's one-block policy (run_max = run_init = 1, no
    format-ahead, slots filled on demand): segments are claimed front first
     even when 148 slots refill at once -- a loser retries among the
    free bits its RMW returned, in the lowest word with free segments -- so
    2^20 16-B requests (16 MB, one segment of slices) stay within the
    segments the concurrent formatters (<= 32 tokens) and the slots' blocks
    take: about one leaf word of 64 segments (bound: 80; round 1's spreading
    over the next words reached 249 segments)."""
    nseg = 1024
    G.gallatin_init(nseg * SEG, run_max=1, run_init=1, format_ahead=2, prefetch=2, prefill=2)
    r = X.fragmentation(16, 1 << 20)
    assert r["nulls"] == 0
    assert r["range_bytes"] < 80 * SEG, f"range {r['range_bytes'] / SEG:.1f} segments"
    G.gallatin_free(r["ptrs"])
    _pristine(G, nseg)


def test_warm_rounds_and_variance(cuda_ok, G, X):
    nseg = 64
    G.gallatin_init(nseg * SEG)
    w = X.warm_vs_cold(64, 1 << 20, rounds=5)
    for k in ("cold", "warm"):
        assert w[k]["malloc_ms"] > 0 and w[k]["free_ms"] > 0 and w[k]["malloc_var_ms2"] >= 0
    v = X.variance(64, 1 << 18, rounds=6)
    assert v["malloc_ms_min"] <= v["malloc_ms_median"] <= v["malloc_ms_max"]
    # the warm state is a correct allocator: a checked round on top of it
    sizes = torch.from_numpy(wg.single_sizes(64, 1 << 20).view(np.int64)).cuda()
    p = G.gallatin_malloc(sizes)
    G.gallatin_stamp(p, sizes)
    assert G.gallatin_verify(p, sizes) == 0
    G.gallatin_free(p)
    _pristine(G, nseg)


def test_init_time_cycles(cuda_ok, G, X):
    r = X.init_time(64 * SEG, reps=2)
    assert r["init_ms_median"] > 0 and not G.gallatin_is_initialized()
    G.gallatin_init(64 * SEG)
    _pristine(G, 64)
