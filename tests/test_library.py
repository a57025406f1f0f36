"""Host-side tests of the C-ABI library (no GPU needed): the library loads and
exports every symbol ``include/fsgc.h`` declares; ``fsgc_compile_pattern``
(host logic) agrees with the oracle's reading of Sec. 3.4; the multi-rank
combine step works over gloo with world_size 2."""
import os
import re
from math import factorial

import pytest

import oracle
from inputs import PATTERNS
from inputs.patterns import all_connected_patterns

F = pytest.importorskip("paper_conf_sc_bradleyab25_b200")
from paper_conf_sc_bradleyab25_b200 import _lib  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "fsgc.h")).read()
    declared = set(re.findall(r"^(?:int|void|const char\s*\*)\s*(fsgc_[a-z_0-9]+)\s*\(", hdr, re.M))
    assert declared, "no declarations parsed"
    for name in declared:
        assert hasattr(_lib.lib, name), name
    assert set(_lib.EXPORTS) == declared
    assert b"sm_100a" in _lib.lib.fsgc_version()


def _check_against_oracle(P):
    p = F.compile_named(P)
    d = oracle.decompose(P.n, P.edges, P.core)
    assert tuple(p.core) == d.core, P
    assert sorted(p.types, key=lambda t: sorted(t[0])) == [(a, k) for a, k in d.types], P
    assert p.aut == oracle.automorphism_count(P.n, P.edges), P
    fact = 1
    for _, k in d.types:
        fact *= factorial(k)
    assert p.fringe_factorial == fact
    # the core-preserving subgroup Aut_C' x prod S_k divides Aut(P)
    assert p.aut % (p.aut_core_labeled * p.fringe_factorial) == 0
    assert p.aut_core % p.aut_core_labeled == 0
    # matching order: connected, starts at a core vertex (Sec. 3.6)
    padj = oracle.pattern_adjacency(P.n, P.edges)
    for i, v in enumerate(p.core_order[1:], 1):
        assert padj[v] & set(p.core_order[:i]), P


def test_compile_matches_oracle_all_small_patterns():
    for P in all_connected_patterns(5):
        _check_against_oracle(P)


def test_compile_matches_oracle_named_patterns():
    for P in PATTERNS.values():
        _check_against_oracle(P)


def test_compile_errors():
    with pytest.raises(F.FsgcError) as e:
        F.fsgc_compile_pattern(4, [(0, 1), (2, 3)])      # disconnected
    assert e.value.code == _lib.FSGC_ERR_PATTERN
    with pytest.raises(F.FsgcError):
        F.fsgc_compile_pattern(3, [(0, 1), (1, 2)], core=[0, 2])   # core not connected
    with pytest.raises(F.FsgcError):
        F.fsgc_compile_pattern(4, [(0, 1), (1, 2), (2, 3)], core=[1])  # fringe 2-3 edge
    with pytest.raises(F.FsgcError):
        F.fsgc_compile_pattern(2, [(0, 0)])             # loop
    with pytest.raises(F.FsgcError):
        F.fsgc_compile_pattern(2, [(0, 1), (1, 0)])     # duplicate


def test_finalize_exact_division():
    assert F.fsgc_finalize(10, 2) == 5
    big = (1 << 127) + 6
    assert F.fsgc_finalize(big, 2) == big // 2
    with pytest.raises(F.FsgcError):
        F.fsgc_finalize(7, 2)
    assert F.fsgc_finalize(6, 2, overflow=True) is None


def _gloo_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # rank r holds a partial raw sum; the true total is divisible by 6
        total = (1 << 100) * 6 + 6 * 12345
        parts = [(1 << 100) * 6 - 17, 6 * 12345 + 17]
        part = [F.CountResult(count=None, raw=parts[rank], divisor=6, core_matches=10 + rank,
                              overflow=False, root_pattern_vertex=0),
                F.CountResult(count=None, raw=(1 << 127) if rank == 0 else (1 << 127), divisor=1,
                              core_matches=0, overflow=False, root_pattern_vertex=0)]
        out = F.combine_partials(part)
        q.put((rank, out[0].count == total // 6, out[0].core_matches, out[1].overflow))
    finally:
        dist.destroy_process_group()


def test_combine_partials_gloo_world2():
    import multiprocessing as mp
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok, cm, ovf in res:
        assert ok and cm == 21 and ovf    # 2^127 + 2^127 overflows 128 bits
