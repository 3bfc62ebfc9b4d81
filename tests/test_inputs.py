"""The seeded input generators (dpgen) are deterministic and shaped like the
workloads of SURVEY.md §8(d)."""
import numpy as np

import dpgen


def test_blosum62_table():
    B = dpgen.blosum62()
    assert B.shape == (24, 24) and (B == B.T).all()
    diag = dict(zip(dpgen.PROTEIN, np.diag(B)))
    assert [diag[c] for c in "ARNDCQEGHILKMFPSTWYV"] == [4, 5, 6, 6, 9, 5, 5, 6, 8, 4, 4, 5, 5, 6, 7, 4, 5, 11, 7, 4]
    assert B.max() == 11 and B[:20, :20].min() == -4
    for a in range(20):  # the diagonal dominates its row among the 20 standard residues
        assert B[a, a] == B[a, :20].max()


def test_pair_mask():
    m = dpgen.rna_pair_mask()
    assert m.sum() == 6 and (m == m.T).all()
    assert dpgen.rna_pair_mask(gu=False).sum() == 4


def test_deterministic_configs():
    a1 = dpgen.config2_protein_pairs(10)
    a2 = dpgen.config2_protein_pairs(10)
    assert all((x == y).all() for x, y in zip(a1, a2))
    assert a1[0].max() < 20 and len(a1[0]) == 2560
    # prefix-consistent sample
    s = dpgen.config2_protein_pairs(3, first=4)
    assert (s[0] == a1[0][4 * 256:7 * 256]).all()
    assert (dpgen.config1_rna64() == dpgen.config1_rna64()).all()
    lens = dpgen.config5_lengths(1000)
    assert lens.min() >= 128 and lens.max() <= 512


def test_config5_subset_matches_full():
    cat, off = dpgen.config5_rna_batch(200)
    ids = [3, 17, 150]
    scat, soff = dpgen.config5_rna_batch(200, ids=ids)
    for k, i in enumerate(ids):
        assert (scat[soff[k]:soff[k + 1]] == cat[off[i]:off[i + 1]]).all()


def test_hmm_config_small():
    d = dpgen.config3_hmm(n_seqs=5, T=50, S=8)
    assert d["A"].shape == (8, 8) and d["E"].shape == (8, 4) and d["seqs"].shape == (5, 50)
    assert np.allclose(d["A"].sum(1), 1, atol=1e-6)
    assert d["lA"].dtype == np.int32 and (d["lA"] <= 0).all()
    assert dpgen.millibits([1.0, 0.5, 0.0]).tolist() == [0, -1000, dpgen.MILLIBIT_FLOOR]
