"""CPU tests of the C-ABI library: it loads, exports every symbol include/uniconn.h declares,
and its host logic (bootstrap allgather, neighbour validation, topology classification,
host barrier) works with virtual ranks and across 2 processes over torch.distributed gloo.
No compute calls (no GPU here)."""
import os
import re
import socket

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

U = pytest.importorskip("paper_conf_cluster_sagbilieinu25_b200")


def _declared():
    hdr = open(os.path.join(ROOT, "include", "uniconn.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(uc_[a-z0-9_]+)\s*\(", hdr)))


def test_exports_every_declared_symbol():
    names = _declared()
    assert len(names) >= 35
    for n in names:
        assert hasattr(U.lib, n), n
    assert set(names) == set(U.EXPORTED)


def test_symbols_in_dynamic_table():
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", U.LIB_PATH], capture_output=True, text=True).stdout
    syms = set(l.split()[-1] for l in out.splitlines() if l.strip())
    for n in _declared():
        assert n in syms, n


def test_build_entry_does_not_import_the_package():
    """__graft_entry__.build() must work on a fresh clone, where importing the package fails
    (no library yet): the builder is loaded by file path."""
    import subprocess
    import sys
    code = ("import sys, __graft_entry__ as g; b = g._builder(); "
            "assert 'paper_conf_cluster_sagbilieinu25_b200' not in sys.modules; print(b.LIB)")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip().endswith("libuniconn_b200.so")


def test_binary_is_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", U.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_enum_constants_match_header():
    hdr = open(os.path.join(ROOT, "include", "uniconn.h")).read()
    for name, val in re.findall(r"\b(UC_[A-Z0-9_]+)\s*=\s*(\d+)", hdr):
        assert getattr(U, name, None) == int(val) or getattr(U._lib, name) == int(val), name
    for name in ("UC_P2P_PINGPONG", "UC_P2P_WINDOW", "UC_P2P_HALO", "UC_MODE_DEVICE", "UC_TOPO_RING", "UC_F64"):
        assert hasattr(U, name), name


def test_status_strings_and_errors():
    assert U.lib.uc_status_string(0) == b"UC_OK"
    assert U.lib.uc_status_string(5) == b"UC_ERR_TIMEOUT"
    with pytest.raises(U.UCError):
        U.Env(2, 1, -1)  # rank out of range
    with pytest.raises(U.UCError):
        U.Env(0, 9, -1)  # more than UC_MAX_RANKS


def _classify(P, neigh):
    from vranks import run_ranks

    def body(r, P, ag):
        env = U.Env(r, P, -1, ag)
        try:
            c = U.Comm(env, *neigh(r, P))
            topo = c.topology
            c.barrier()
            c.destroy()
            return topo
        finally:
            env.finalize()

    return run_ranks(P, body, timeout=60)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_topology_classification_virtual_ranks(P):
    assert _classify(P, U.ring_neighbours) == [U.UC_TOPO_RING] * P
    assert _classify(P, U.chain_neighbours) == [U.UC_TOPO_CHAIN] * P
    assert _classify(P, lambda r, P: (-1, -1)) == ([U.UC_TOPO_CHAIN] if P == 1 else [U.UC_TOPO_NONE] * P)


def test_inconsistent_neighbours_rejected():
    with pytest.raises(U.UCError, match="UC_ERR_ARG"):
        _classify(3, lambda r, P: ((r + 1) % P, (r + 1) % P))


def test_env_state_errors():
    env = U.Env(0, 1, -1)
    c = U.Comm(env, 0, 0)
    with pytest.raises(U.UCError, match="UC_ERR_STATE"):
        env.finalize()  # communicator still alive
    with pytest.raises(U.UCError, match="UC_ERR_STATE"):
        U.SymMem(c, 1024)  # bootstrap-only env has no device
    with pytest.raises(U.UCError, match="UC_ERR_STATE"):
        U.Jacobi(c, 64, 64)
    c.destroy()
    env.finalize()


# ------------------------------------------------------------------ 2 processes over gloo
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _gloo_worker(rank, world, port, q):
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        import paper_conf_cluster_sagbilieinu25_b200 as UU
        out = {}
        for name, neigh in (("ring", UU.ring_neighbours), ("chain", UU.chain_neighbours)):
            env = UU.Env(rank, world, -1, UU.torch_allgather())
            c = UU.Comm(env, *neigh(rank, world))
            out[name] = (c.rank, c.size, c.top, c.bottom, c.topology)
            c.barrier()
            c.destroy()
            env.finalize()
        env = UU.Env(rank, world, -1, UU.torch_allgather())
        try:
            UU.Comm(env, rank, -1)  # self as top: inconsistent
            out["bad"] = "accepted"
        except UU.UCError as e:
            out["bad"] = "UC_ERR_ARG" in str(e)
        env.finalize()
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_gloo_two_process_bootstrap():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert res[0]["ring"] == (0, 2, 1, 1, U.UC_TOPO_RING)
    assert res[1]["ring"] == (1, 2, 0, 0, U.UC_TOPO_RING)
    assert res[0]["chain"] == (0, 2, -1, 1, U.UC_TOPO_CHAIN)
    assert res[1]["chain"] == (1, 2, 0, -1, U.UC_TOPO_CHAIN)
    assert res[0]["bad"] is True and res[1]["bad"] is True
