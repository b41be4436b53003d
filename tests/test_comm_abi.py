"""CPU-only: the communicator / placement part of the C ABI (e3.h "comm",
e3_plan.replicas / device_of / transport) validates before any launch and
needs no GPU for the loopback handles or the NCCL unique id."""
import ctypes as C

import pytest

import e3data


@pytest.fixture(scope="module")
def L():
    from paper_conf_sosp_iyergdpgn24_b200 import _lib, api
    return _lib, api


def _weights(_lib, n_layers=4, n_ramps=2):
    lw = (_lib.LayerWeights * n_layers)()
    rw = (_lib.RampWeights * n_ramps)()
    return _lib.Weights(n_layers, lw, n_ramps, rw), lw, rw


def _create(_lib, plan, comm, device=0):
    w, lw, rw = _weights(_lib)
    h = C.c_void_p()
    st = _lib.lib.e3_pipeline_create(C.byref(plan), C.byref(w), device, comm.h if comm else None, C.byref(h))
    return st, _lib.lib.e3_last_error().decode()


def test_loopback_comm_handles(L):
    _lib, api = L
    cs = api.Comm.loopback(3, 0)
    assert [c.rank_world() for c in cs] == [(0, 3), (1, 3), (2, 3)]
    for c in cs:
        c.close()


def test_unique_id_is_nccl_sized_or_reports_enccl(L):
    _lib, api = L
    buf = C.create_string_buffer(_lib.E3_COMM_ID_BYTES)
    st = _lib.lib.e3_comm_unique_id(buf)
    assert st in (0, 4)                      # E3_OK, or E3_ENCCL without a usable NCCL
    if st == 4:
        assert b"NCCL" in _lib.lib.e3_last_error() or b"nccl" in _lib.lib.e3_last_error()


def test_plan_placement_validation_before_any_launch(L):
    _lib, api = L
    cfg = e3data.get("tiny")
    cs = api.Comm.loopback(3, 0)
    ok = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0], [1]], transport="loopback")
    # replicas without a communicator
    assert _create(_lib, ok, None)[0] == 1
    # transport mismatch with the communicator
    bad = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0], [1]], transport="nccl")
    st, msg = _create(_lib, bad, cs[0])
    assert st == 1 and "transport" in msg
    # P2P is reserved
    bad = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0], [1]], transport="p2p")
    assert _create(_lib, bad, cs[0])[0] == 2
    # a rank in two stages (non-adjacent split ranges would need two queues)
    bad = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0, 1], [1]], transport="loopback")
    st, msg = _create(_lib, bad, cs[0])
    assert st == 1 and "disjoint" in msg
    # a rank outside the communicator, duplicate replicas
    bad = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0], [5]], transport="loopback")
    assert _create(_lib, bad, cs[0])[0] == 1
    bad = api.make_plan(cfg, (0, 2, 4), cfg.tau, placement=[[0, 0], [1]], transport="loopback")
    assert _create(_lib, bad, cs[0])[0] == 1
    # the plan must end in the model's final ramp
    bad = api.make_plan(cfg, (0, 2), cfg.tau, placement=[[0]], transport="loopback")
    st, msg = _create(_lib, bad, cs[0])
    assert st == 1 and "final" in msg
    # device differs from the communicator's
    assert _create(_lib, ok, cs[0], device=1)[0] == 1
    # dependent exits keep per-input state in the caller's records: one rank only
    pcfg = e3data.get("tp")
    bad = api.make_plan(pcfg, (0, 2, 4), pcfg.tau, placement=[[0], [1]], transport="loopback")
    st, msg = _create(_lib, bad, cs[0])
    assert st == 2 and "single-rank" in msg
    for c in cs:
        c.close()
