"""GPU parity: the CUDA library (through the C ABI) against the CPU oracle, end by end, bit-exact
(extension string, termination code, k of the returned walk, attempts) — DESIGN.md §5.

All inputs are seeded and synthetic (gen/); expected values come only from oracle/ or from closed
forms of the constructions.
"""
import os

import numpy as np
import pytest

from conftest import cached_batch
from gen import Params
from gen import cases as C

pytestmark = pytest.mark.gpu

P0 = Params()


@pytest.fixture(scope="module")
def LA():
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    la = LocalAssembler(0)
    yield la
    la.close()


def check(LA, orc, batch, P, ends=None, env=None):
    old = {}
    for k, v in (env or {}).items():
        old[k] = os.environ.get(k)
        os.environ[k] = v
    try:
        r = LA.load(batch, P).extend()
        st = LA.stats()
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    ref = orc.extend(batch, P, ends=ends)
    sel = ref["ends"]
    got = r.ext_list()
    bad = [int(e) for i, e in enumerate(sel) if got[e] != ref["ext"][i]
           or r.term[e] != ref["term"][i] or r.k_used[e] != ref["k_used"][i]
           or r.n_attempts[e] != ref["n_attempts"][i]]
    if bad:
        e = bad[0]
        i = int(np.nonzero(sel == e)[0][0])
        raise AssertionError(
            f"{len(bad)}/{len(sel)} ends differ; first end {e}: gpu=({got[e][:40]}..., len {len(got[e])}, "
            f"term {r.term[e]}, k {r.k_used[e]}, att {r.n_attempts[e]}) oracle=({ref['ext'][i][:40]}..., len "
            f"{len(ref['ext'][i])}, term {ref['term'][i]}, k {ref['k_used'][i]}, att {ref['n_attempts'][i]})")
    if ends is None:
        assert st["inserts"] == int(ref["inserts"].sum())
        assert st["walk_steps"] == int(ref["walk_steps"].sum())
        assert st["ext_bases"] == sum(len(x) for x in ref["ext"])
    return r, st


def test_c1_single_k(LA, orc):
    check(LA, orc, cached_batch("C1"), Params(k_start=21, k_min=21, k_max=21))


def test_c2_small_full_schedule(LA, orc):
    r, st = check(LA, orc, cached_batch("C2", scale=0.03), P0)
    assert st["ends_by_class"][2] > 0 and st["ends_medium"] > 0 and st["ends_xl"] > 0


def test_c2_small_forced_global(LA, orc):
    _, st = check(LA, orc, cached_batch("C2", scale=0.03), P0, env={"LA_FORCE_GLOBAL": "1"})
    assert st["ends_by_class"][2] == 0 and st["ends_by_class"][3] > 0


def test_c2_small_forced_overflow(LA, orc):
    """Route everything to shared memory: ends whose tables overflow are redone in global memory."""
    _, st = check(LA, orc, cached_batch("C2", scale=0.03), P0, env={"LA_FORCE_SMEM": "1"})
    assert st["ends_by_class"][4] > 0


@pytest.mark.parametrize("P", [
    Params(k_start=25, k_min=17, k_max=45, k_shift=4, max_walk_len=120, q_lo=5, q_hi=30, min_votes=3,
           min_frac_pct=30),
    Params(k_start=31, k_min=31, k_max=128, k_shift=16, min_votes=1, min_frac_pct=0),
    Params(k_start=64, k_min=32, k_max=96, k_shift=32, max_walk_len=1024),
    Params(k_start=9, k_min=5, k_max=13, k_shift=2, max_walk_len=50),
    Params(max_walk_len=0),
])
def test_c2_small_params(LA, orc, P):
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(300))
    check(LA, orc, b, P)


def test_c3_sampled(LA, orc):
    """High-skew workload: every hot end (global path) and a sample of sparse ends."""
    b = cached_batch("C3")
    r = b.reads_per_end()
    hot = np.nonzero(r >= 10000)[0][:3]
    rng = np.random.default_rng(0)
    ends = np.concatenate([hot, rng.choice(b.n_ends, 300, replace=False)])
    _, st = check(LA, orc, b, P0, ends=ends)
    assert st["ends_by_class"][3] >= len(hot)


def test_pins_on_gpu(LA, orc):
    """Closed-form constructions (P2-P8) through the GPU path, batched as one multi-contig batch."""
    rng = np.random.default_rng(1)
    G = C.unique_genome(rng, 1200)
    contigs, ends = [], []
    # P2 DEADEND chain, P6 MAXLEN, P7 N in contig, P8 NOREADS/SHORT/short reads
    for e, a_hi in ((500, 600), (500, 1000)):
        contigs.append(G[e - 200:e]); ends += [C.tile(G, 0, 250, 150, qchar="5"), C.tile(G, 200, a_hi, 150)]
    nc = list(G[300:500]); nc[200 - 1 - 27] = "N"
    contigs.append("".join(nc)); ends += [[], C.tile(G, 200, 600, 150)]
    contigs.append(G[468:500]); ends += [[], C.tile(G, 200, 600, 150)]
    contigs.append(G[300:500]); ends += [[], [(s[:21], q[:21]) for s, q in C.tile(G, 200, 600, 150)]]
    u = 110
    while True:
        U, FL, FR = C.random_seq(rng, u), C.random_seq(rng, 200), C.random_seq(rng, 200)
        if C.kmers_unique(FL + U + FR, 21):
            break
    reg = FL + U * 7 + FR
    contigs.append(reg[300:580]); ends += [[], C.tile(reg, 0, len(reg) - 150, 150)]
    b = C.Batch.from_lists(contigs, ends)
    r, _ = check(LA, orc, b, P0)
    assert r.ext(1) == G[500:749] and r.term[1] == 0
    assert r.ext(3) == G[500:800] and r.term[3] == 3
    assert r.k_used[5] == 25
    assert r.term[6] == 4 and r.term[7] == 5
    assert r.ext(9) == "" and r.term[9] == 0
    assert r.ext(11) == reg[580:690] and r.term[11] == 2


def test_rc_twin_and_permutation(LA, orc):
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(200))
    r = LA.load(b, P0).extend()
    ext = r.ext_list()
    tw = C.twin(b)
    rt = LA.load(tw, P0).extend()
    ext_t = rt.ext_list()
    for c in range(b.n_contigs):
        assert ext_t[2 * c] == C.rc(ext[2 * c + 1]) and ext_t[2 * c + 1] == C.rc(ext[2 * c])
    bp, perm = C.permuted(b, 5)
    rp = LA.load(bp, P0).extend()
    idx = np.stack([2 * perm, 2 * perm + 1], 1).reshape(-1)
    assert [ext[i] for i in idx] == rp.ext_list()
    assert np.array_equal(r.term[idx], rp.term)


def test_device_memory_input(LA, orc):
    import torch
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(150))
    host = LA.load(b, P0).extend()

    class DevBatch:
        pass
    d = DevBatch()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
        setattr(d, f, torch.from_numpy(getattr(b, f)).cuda())
    dev = LA.load(d, P0).extend()
    assert host.ext_list() == dev.ext_list() and np.array_equal(host.term, dev.term)


def test_empty_and_degenerate(LA, orc):
    check(LA, orc, C.Batch.from_lists([], []), P0)
    check(LA, orc, C.Batch.from_lists(["ACGT" * 10, "A"], [[], [], [], []]), P0)
    # reads of length 0 and reads of only N
    check(LA, orc, C.Batch.from_lists(["ACGT" * 20], [[("", "")], [("N" * 150, "I" * 150)]]), P0)


def test_invalid_inputs_leave_context_unchanged(LA, orc):
    from paper_conf_sc_awanhedbdoy21_b200._lib import LocAssmError
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(50))
    good = LA.load(b, P0).extend().ext_list()
    bad = C.Batch.from_lists(["ACGTX" * 10], [[], []])
    with pytest.raises(LocAssmError, match="INVALID_ARG"):
        LA.load(bad, P0)
    bad2 = C.Batch.from_lists(["ACGT" * 10], [[], [("A" * 301, "I" * 301)]])
    with pytest.raises(LocAssmError, match="300"):
        LA.load(bad2, P0)
    bad3 = C.Batch.from_lists(["ACGT" * 10], [[], [("ACGT", "I!II")]])
    with pytest.raises(LocAssmError, match="qual"):
        LA.load(bad3, P0.replace(qual_offset=40))
    with pytest.raises(LocAssmError, match="k schedule"):
        LA.load(b, P0.replace(k_start=10))
    assert LA.extend().ext_list() == good


def test_state_error_before_load():
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    from paper_conf_sc_awanhedbdoy21_b200._lib import LocAssmError
    with LocalAssembler(0) as la:
        with pytest.raises(LocAssmError, match="STATE"):
            la.extend()


@pytest.fixture(scope="module")
def c2_ref(orc):
    b = cached_batch("C2", scale=0.03)
    return b, orc.extend(b, P0)


@pytest.mark.parametrize("n_chunks", [1, 3, 8, 4000])
def test_streamed_matches_oracle(LA, c2_ref, n_chunks):
    """la_extend_streamed (NEXT N1): chunked host batch, copies overlapped with extension — every end
    bit-exact against the oracle, work counters summed over chunks; 4000 chunks > contigs."""
    b, ref = c2_ref
    r = LA.extend_streamed(b, P0, n_chunks)
    st = LA.stats()
    assert r.ext_list() == ref["ext"]
    for f in ("term", "k_used", "n_attempts"):
        assert np.array_equal(getattr(r, f), ref[f]), f
    assert st["inserts"] == int(ref["inserts"].sum())
    assert st["walk_steps"] == int(ref["walk_steps"].sum())
    # the context stays usable for the ordinary load + extend path
    assert LA.load(b.select_contigs(np.arange(20)), P0).extend().n_ends == 40


def test_streamed_edge_cases(LA, orc):
    from paper_conf_sc_awanhedbdoy21_b200._lib import LocAssmError
    import torch
    empty = C.Batch.from_lists([], [])
    assert LA.extend_streamed(empty, P0, 4).n_ends == 0
    small = C.Batch.from_lists(["ACGT" * 20, "A"], [[("N" * 150, "I" * 150)], [], [], []])
    ref = orc.extend(small, P0)
    r = LA.extend_streamed(small, P0, 2)
    assert r.ext_list() == ref["ext"] and np.array_equal(r.term, ref["term"])
    with pytest.raises(LocAssmError, match="n_chunks"):
        LA.extend_streamed(small, P0, 0)
    bad = C.Batch.from_lists(["ACGT" * 10, "ACGTX" * 10], [[], [], [], []])
    with pytest.raises(LocAssmError, match="INVALID_ARG"):
        LA.extend_streamed(bad, P0, 2)

    class DevBatch:
        pass
    d = DevBatch()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
        setattr(d, f, torch.from_numpy(getattr(small, f)).cuda())
    with pytest.raises(LocAssmError, match="host batch"):
        LA.extend_streamed(d, P0, 2)


@pytest.mark.parametrize("k_start", [21, 55, 77])
def test_assembler_k_rounds(LA, orc, k_start):
    """NEXT N2: local assembly at the other k of the assembler's contig iteration (Fig 1 "iterate
    for k"); k_start 77 starts on pointer (REF) keys, 55 upshifts into them."""
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(400))
    check(LA, orc, b, P0.replace(k_start=k_start, k_min=21, k_max=99))


def _appended_strings(seq, off):
    b = seq.cpu().numpy().tobytes()
    o = off.cpu().numpy()
    return [b[o[i]:o[i + 1]].decode() for i in range(o.shape[0] - 1)]


def test_append_extensions_matches_oracle(LA, c2_ref):
    """la_append_extensions (NEXT N1, Fig 4 "Append extensions to contigs"): device pipeline
    load -> extend_device -> append, every extended contig equal to the oracle's
    ext[2c] + contig + ext[2c+1]."""
    import torch
    import oracle
    b, ref = c2_ref
    contigs = [b.contig_seq[b.contig_off[c]:b.contig_off[c + 1]].tobytes().decode() for c in range(b.n_contigs)]
    want = oracle.append_extensions(contigs, ref["ext"])
    cseq = torch.from_numpy(b.contig_seq).cuda()
    coff = torch.from_numpy(b.contig_off).cuda()
    d = LA.load(b, P0).extend_device()
    seq, off = LA.append_extensions(cseq, coff, d["ext_off"], d["ext_seq"])
    assert int(off[0]) == 0 and int(off[-1]) == sum(len(x) for x in want)
    assert _appended_strings(seq, off) == want


def test_append_extensions_edge_cases(LA):
    """Offsets not starting at 0 (a slice of a larger batch), empty extensions and contigs, none."""
    import torch
    import oracle
    contigs = ["ACGTACGT", "", "GATTACA", "T"]
    ext = ["CC", "", "A", "TTT", "", "", "G", "NACG"]
    cseq = torch.tensor(list(b"XXXX" + "".join(contigs).encode()), dtype=torch.uint8).cuda()
    coff = torch.tensor([4 + sum(len(x) for x in contigs[:i]) for i in range(5)], dtype=torch.int64).cuda()
    eseq = torch.tensor(list(b"ZZ" + "".join(ext).encode()), dtype=torch.uint8).cuda()
    eoff = torch.tensor([2 + sum(len(x) for x in ext[:i]) for i in range(9)], dtype=torch.int64).cuda()
    seq, off = LA.append_extensions(cseq, coff, eoff, eseq)
    assert _appended_strings(seq, off) == oracle.append_extensions(contigs, ext)
    z = torch.zeros(1, dtype=torch.int64).cuda()
    seq, off = LA.append_extensions(torch.zeros(0, dtype=torch.uint8).cuda(), z, z,
                                    torch.zeros(0, dtype=torch.uint8).cuda())
    assert seq.numel() == 0 and off.tolist() == [0]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_append_extensions_alignments(LA, seed):
    """Random segment lengths 0..300 and random leading offsets, so every source/destination
    alignment (the 16-byte realigned copy, heads and tails) is exercised; against the oracle."""
    import torch
    import oracle
    rng = np.random.default_rng(100 + seed)
    n = 700

    def rs(m):
        return "".join(rng.choice(list("ACGTN"), m)) if m else ""
    contigs = [rs(int(rng.integers(0, 300))) for _ in range(n)]
    ext = [rs(int(rng.integers(0, 300)) if rng.random() < 0.8 else 0) for _ in range(2 * n)]
    pc, pe = int(rng.integers(0, 16)), int(rng.integers(0, 16))
    cseq = torch.tensor(list(b"x" * pc + "".join(contigs).encode()), dtype=torch.uint8).cuda()
    eseq = torch.tensor(list(b"y" * pe + "".join(ext).encode()), dtype=torch.uint8).cuda()
    coff = torch.from_numpy(pc + np.concatenate([[0], np.cumsum([len(x) for x in contigs])])).cuda()
    eoff = torch.from_numpy(pe + np.concatenate([[0], np.cumsum([len(x) for x in ext])])).cuda()
    seq, off = LA.append_extensions(cseq, coff, eoff, eseq)
    assert _appended_strings(seq, off) == oracle.append_extensions(contigs, ext)


@pytest.mark.parametrize("cls", range(7))
def test_class_by_key_format_matrix(LA, orc, cls):
    """Every table class (0-4 shared memory, 5 = XL in global scratch, 6 = XLC split over a 2-CTA
    cluster) with inline keys (k <= 63) and pointer keys (k >= 64), each forced (LA_FORCE_CLASS) and
    compared with the oracle end by end.  XLC builds inline keys only: its ends with a k >= 64 attempt
    are redone by the global rounds (still bit-exact)."""
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(400))
    for P, key in ((P0, "cls_inl_attempts"), (Params(k_start=65, k_min=57, k_max=97), "cls_ref_attempts")):
        _, st = check(LA, orc, b, P, env={"LA_FORCE_CLASS": str(cls)})
        if cls == 6 and key == "cls_ref_attempts":   # k 65 first: every end goes on to the global rounds
            assert st["ends_by_class"][4] > 0
        else:
            assert st[key][cls] > 0, (cls, key, st[key])


def test_xlc_cluster_class(LA, orc):
    """XLC (2-CTA cluster, table in both SMs' shared memory): C3's densest non-hot ends and the C2 slice
    forced into it, bit-exact; and the planner routes ends there on its own."""
    b = cached_batch("C2", scale=0.03)
    _, st = check(LA, orc, b, P0, env={"LA_FORCE_CLASS": "6"})
    assert st["cls_ends"][6] > 0 and st["cls_inl_attempts"][6] > 0
    _, st = check(LA, orc, b, P0)
    assert st["cls_ends"][6] == 0   # opt-in (LA_XLC=1): not planned by default


def test_replay_build_reruns_the_attempts(LA, orc):
    """la_replay_build reruns exactly the extension's table builds (same inserts) and leaves its
    results unchanged; attempts_hist counts every end."""
    b = cached_batch("C2", scale=0.03)
    r, st = check(LA, orc, b, P0)
    rp = LA.replay_build()
    assert sum(rp["cls_build_inserts"]) == st["inserts_smem"]
    assert rp["ms_build"] > 0 and rp["ms_walk"] == pytest.approx(st["ms_smem"] - rp["ms_build"])
    assert sum(st["attempts_hist"]) == b.n_ends
    assert st["attempts_hist"] == np.bincount(np.minimum(r.n_attempts, 15), minlength=16).tolist()
    r2 = LA.extend()
    assert r2.ext_list() == r.ext_list() and np.array_equal(r2.term, r.term)


def test_c_abi_client():
    """The plain C client (examples/abi_client.c) on the device: closed-form pin P2 through the ABI, and
    the N4 selection's closed-form count followed by the extension of the selected device batch."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import __graft_entry__
    __graft_entry__.build()   # (re)builds the client against the current header and library
    exe = os.path.join(root, "examples", "abi_client")
    out = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    assert out.stdout.count("abi_client ok") == 2, out.stdout


def test_xl_wide_counters(LA, orc):
    """XL tables with 32-bit counter fields: an end with >= 65536 voting occurrences per attempt (700
    reads of a 20,000x end of C3) forced into the XL class; and the same end's first 300 reads (16-bit
    fields).  Both against the oracle."""
    b = cached_batch("C3")
    r = b.reads_per_end()
    e = int(np.nonzero(r >= 10000)[0][0])
    c = e // 2
    contig = b.contig_seq[b.contig_off[c]:b.contig_off[c + 1]].tobytes().decode()

    def reads(n):
        out = []
        for j in range(b.end_read_off[e], b.end_read_off[e] + n):
            s0, s1 = b.read_off[j], b.read_off[j + 1]
            out.append((b.read_seq[s0:s1].tobytes().decode(), b.read_qual[s0:s1].tobytes().decode()))
        return out
    for n in (700, 300):
        ends = [[], reads(n)] if e % 2 else [reads(n), []]
        sub = C.Batch.from_lists([contig], ends)
        _, st = check(LA, orc, sub, P0, env={"LA_FORCE_CLASS": "5"})
        assert st["cls_inl_attempts"][5] > 0 and st["ends_by_class"][4] == 0


@pytest.mark.parametrize("share", [1.0, 0.3])
def test_coexec_matches_oracle(LA, orc, share):
    """NEXT N3: the lightest ends of the smallest class extended on host threads while the GPU runs
    (la_set_coexec) — every end still bit-exact against the oracle, work counters included."""
    b = cached_batch("C2", scale=0.03)
    LA.set_coexec(8, share)
    try:
        r, st = check(LA, orc, b, P0)
    finally:
        LA.set_coexec(0, 0.0)
    assert st["cpu_ends"] > 0 and st["cpu_inserts"] > 0
    r2 = LA.extend()   # co-execution off: same results, no host ends
    assert r2.ext_list() == r.ext_list() and LA.stats()["cpu_ends"] == 0


def test_coexec_streamed(LA, orc, c2_ref):
    b, ref = c2_ref
    LA.set_coexec(4, 0.5)
    try:
        r = LA.extend_streamed(b, P0, 3)
        st = LA.stats()
    finally:
        LA.set_coexec(0, 0.0)
    assert r.ext_list() == ref["ext"] and np.array_equal(r.term, ref["term"])
    assert st["cpu_ends"] > 0 and st["inserts"] == int(ref["inserts"].sum())
