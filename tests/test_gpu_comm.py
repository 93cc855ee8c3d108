"""The strata mode's transport primitives (a12: Q rotation by grouped send/recv, the RMSE
all-reduce, the segment gather of mf_get_factors; section 6.1, P:L305-316 adapted) run and
checked through mf_comm_selftest.  On the one GPU a test box has, world = 1 executes every NCCL
call the multi-GPU epoch makes (the rotation as a send/recv to self); the loopback transport runs
the same primitives with 2 and 4 ranks as threads."""
import os
import threading

import pytest

from paper_conf_hpdc_xietfl17_b200 import mf

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)


def test_nccl_primitives_execute_on_one_gpu(capfd):
    uid = mf._nccl_get_unique_id()
    rep = mf.comm_selftest(uid, world=1, rank=0, device=0, transport=0)
    assert rep.startswith("ok: NCCL, rank 0 of 1"), rep
    err = capfd.readouterr().err
    assert "[mf_comm] NCCL communicator ready: rank 0 of 1, ncclCommCount = 1" in err, err


@pytest.mark.parametrize("world", [1, 2, 4])
def test_loopback_primitives_with_rank_threads(world):
    key = os.urandom(16)
    out, errs = [None] * world, []

    def rank_main(r):
        try:
            out[r] = mf.comm_selftest(key, world=world, rank=r, device=0, transport=1)
        except Exception as e:  # noqa: BLE001 -- reported below
            errs.append(e)

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=120)
    assert not errs, errs
    assert all(o and o.startswith(f"ok: loopback, rank {r} of {world}") for r, o in enumerate(out)), out
