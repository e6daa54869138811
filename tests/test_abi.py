"""CPU checks of the C-ABI boundary: librp.so loads without a GPU and exports every
function include/rp.h declares; host-side argument validation works without a device."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "rp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(rp_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("rp_create", "rp_destroy", "rp_history_init", "rp_deposit_step",
                 "rp_compute_potentials", "rp_compute_fields", "rp_push_particles"):
        assert must in names


def test_library_exports_every_declared_symbol():
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    lib = C.CDLL(rp.LIB_PATH)
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing
    # and the binding wraps every one of them under the same name
    assert sorted(rp.EXPORTED) == _declared()
    for n in _declared():
        assert callable(getattr(rp, n))


def test_host_side_calls_without_gpu():
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    assert rp.rp_version() == 200
    assert rp.rp_strerror(0) == "ok"
    assert rp.rp_strerror(-5) == "call out of order"
    # invalid configurations are rejected before any device call
    with pytest.raises(rp.RpError) as e:
        rp.rp_create(3, 32, 1.0, 1.0, 10, 1.0, 1.0, 1e-6)
    assert e.value.code == -1
    with pytest.raises(rp.RpError) as e:
        rp.rp_create(32, 32, 1.0, 1.0, 10, 1.0, 1.0, 1e-6, n_theta=63)
    assert e.value.code == -1
    with pytest.raises(rp.RpError) as e:
        rp.rp_create(32, 32, 1.0, 1.0, 10, 1.0, 1.0, 1e-6, n_root=3)
    assert e.value.code == -1
    assert rp.rp_shard_capacity(None, 2) == 0
    # multi-GPU membership is validated before any device call: rank outside [0, world)
    nid = bytes(rp.RP_NCCL_ID_BYTES)
    for rank, world in ((2, 2), (-1, 2), (0, 0)):
        with pytest.raises(rp.RpError) as e:
            rp.rp_create(32, 32, 1.0, 1.0, 10, 1.0, 1.0, 1e-6, dist=(rank, world, nid))
        assert e.value.code == -1
    with pytest.raises(ValueError):
        rp.rp_create(32, 32, 1.0, 1.0, 10, 1.0, 1.0, 1e-6, dist=(0, 1, b"short"))
    assert rp.rp_strerror(-4).startswith("NCCL")
    # setters reject bad arguments on a NULL context before touching it
    with pytest.raises(rp.RpError):
        rp.rp_set_work_split(None, 5)
    with pytest.raises(rp.RpError):
        rp.rp_set_work_split(None, 5, 3)


def test_nccl_unique_id_loads_nccl_at_run_time():
    """librp resolves NCCL with dlopen (no link-time dependency): a unique id for rp_dist can
    be made on a host without a GPU."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    try:
        a = rp.rp_nccl_unique_id()
    except rp.RpError as e:  # pragma: no cover - an image without libnccl
        assert e.code == -4
        pytest.skip("libnccl.so.2 not loadable here")
    b = rp.rp_nccl_unique_id()
    assert len(a) == rp.RP_NCCL_ID_BYTES and a != b
