"""Host logic of the time series' per-scan resumability: the
result store writes each grid's records atomically, lists what is done, and `pending` keeps
the order of the indices still to run.  (The resume itself on the GPU: test_gpu_parity.)"""
import os

import numpy as np

from paper_conf_icpp_blattnerkcsbz14_b200 import PAIR_DTYPE
from paper_conf_icpp_blattnerkcsbz14_b200.stream import GridResult, ResultStore, pending


def result(i, n=3, m=4):
    rng = np.random.default_rng(i)
    w = np.zeros((n, m), PAIR_DTYPE)
    no = np.zeros((n, m), PAIR_DTYPE)
    for a in (w, no):
        a["dx"] = rng.integers(-50, 50, (n, m))
        a["dy"] = rng.integers(-50, 50, (n, m))
        a["ccf"] = rng.random((n, m))
        a["candidate"] = rng.integers(0, 5, (n, m))
    return GridResult(i, w, no)


def test_store_round_trip_and_done(tmp_path):
    st = ResultStore(str(tmp_path / "s"))
    assert st.done() == set()
    for i in (0, 3, 17):
        st.save(result(i))
    assert st.done() == {0, 3, 17}
    r = st.load(3)
    ref = result(3)
    assert r.index == 3 and r.west.tobytes() == ref.west.tobytes() and \
        r.north.tobytes() == ref.north.tobytes()
    st.save(result(3))                      # overwrite in place (a re-run of one grid)
    assert st.done() == {0, 3, 17}


def test_store_ignores_partial_and_foreign_files(tmp_path):
    st = ResultStore(str(tmp_path / "s"))
    st.save(result(1))
    # a crash mid-write leaves only a temporary file; unrelated files are ignored
    open(os.path.join(st.dir, ".tmp_2_123.npz"), "wb").write(b"partial")
    open(os.path.join(st.dir, "grid_notanumber.npz"), "wb").write(b"x")
    open(os.path.join(st.dir, "notes.txt"), "w").write("x")
    assert st.done() == {1}


def test_pending_keeps_order_and_skips_done(tmp_path):
    st = ResultStore(str(tmp_path / "s"))
    assert pending(range(5), None) == [0, 1, 2, 3, 4]
    assert pending([4, 2, 0, 3], st) == [4, 2, 0, 3]
    for i in (2, 3):
        st.save(result(i))
    assert pending(range(6), st) == [0, 1, 4, 5]
    assert pending([3, 2], st) == []
