"""Seeded generators (no method arithmetic): the C4F Fig 3 mix and the N4 read pool."""
import numpy as np

from gen import make
from gen.pool import make_pool


def test_c4f_has_the_fig3_mix_and_keeps_read_prefixes():
    """C4F (Fig 3): ~70% of ends without reads, 10-30% with 1-9, < 1% with >= 10; every
    kept read set is a prefix of the same end's C4 reads (same contigs, same order)."""
    full = make("C4", scale=0.01)
    sub = make("C4F", scale=0.01)
    assert np.array_equal(sub.contig_off, full.contig_off) and np.array_equal(sub.contig_seq, full.contig_seq)
    r, rf = sub.reads_per_end(), full.reads_per_end()
    assert 0.65 < (r == 0).mean() < 0.75
    assert 0.10 <= ((r > 0) & (r < 10)).mean() <= 0.30
    assert (r >= 10).mean() < 0.012
    assert (r <= rf).all()
    for e in np.nonzero(r)[0][:200]:
        a = sub.read_off[sub.end_read_off[e]:sub.end_read_off[e + 1] + 1]
        b = full.read_off[full.end_read_off[e]:full.end_read_off[e] + r[e] + 1]
        assert sub.read_seq[a[0]:a[-1]].tobytes() == full.read_seq[b[0]:b[-1]].tobytes()


def test_pool_pairs_are_fr_and_match_the_truth():
    """FR pairs: mate 0 is G[f, f+L) when strand 0, else rc of the fragment's last L bases (and mate 1
    the other), from the truth coordinates, error-free."""
    p = make_pool(seed=3, genome_len=5000, n_contigs=3, coverage=5, err=0.0, n_rate=0.0)
    G = np.frombuffer(b"ACGT", np.uint8)[p.truth["genome"]].tobytes()
    comp = bytes.maketrans(b"ACGT", b"TGCA")
    s = p.read_seq.tobytes()
    for i in range(p.n_pairs):
        f, ins, z = int(p.truth["frag_start"][i]), int(p.truth["ins"][i]), int(p.truth["strand"][i])
        fwd, rev = G[f:f + 150], G[f + ins - 150:f + ins][::-1].translate(comp)
        m0, m1 = s[300 * i:300 * i + 150], s[300 * i + 150:300 * i + 300]
        assert (m0, m1) == ((fwd, rev) if z == 0 else (rev, fwd))
