"""Worked-example fixtures of the paper, as GFSL pool images.

A fixture lists each level's chunks left to right; chunk entries are user keys
("-inf" for the first chunk's sentinel) with, above level 0, the name of the chunk their
down pointer targets.  Chunk 0 of every level is that level's head chunk of a fresh
structure; the others are allocated in order from the right pool (R18).
Figures and their pinned facts are cited in tests/test_oracle_b.py.
"""
from oracle.oracle_b import E, EMPTY, FREE, GFSLModel, INF, NEG_INF, NULL

# Fig 4.1, N = 6 (DSIZE 4).  Level 2: A; level 1: B, C; level 0: E0..L
FC = {
    2: [("A", [("-inf", "B"), (59, "C")])],
    1: [("B", [("-inf", "E0"), (10, "E"), (30, "G"), (47, "H")]),
        ("C", [(59, "I"), (68, "J"), (75, "K"), (80, "L")])],
    0: [("E0", [3, 6]), ("E", [10, 13, 17, 21]), ("F", [24, 26]), ("G", [30, 33, 40]),
        ("H", [47, 50]), ("I", [59, 63]), ("J", [68, 71]), ("K", [75, 77]), ("L", [80, 90])],
}
# level 0 of a non-first chunk has no -inf; E0 (the first) gets -inf prepended below

# Fig 4.2/4.3: FC with E = [10, 17, 21]
FI = {l: list(v) for l, v in FC.items()}
FI[0] = [(n, ([10, 17, 21] if n == "E" else ks)) for n, ks in FC[0]]

# Fig 4.4, N = 6: a full bottom chunk B split by inserting 22
FS = {
    1: [("A", [("-inf", "B"), (20, "B")])],
    0: [("B", [12, 20, 25])],          # with -inf: [-inf, 12, 20, 25] (full at DSIZE 4)
}

# Fig 4.5, N = 12 (DSIZE 10, merge threshold 3)
FD = {
    2: [("A", [("-inf", "B"), (24, "B")])],
    1: [("B", [("-inf", "E0"), (13, "E"), (24, "F")])],
    0: [("E0", [5, 8]), ("E", [13, 17, 21]), ("F", [24, 26])],
}
# Fig 4.6: no merge, E = [13, 17, 21, 22]
FDN = {l: list(v) for l, v in FD.items()}
FDN[0] = [("E0", [5, 8]), ("E", [13, 17, 21, 22]), ("F", [24, 26])]


def build(spec, N, key_range=100, cap_bottom=64, cap_upper=64):
    """A GFSLModel holding the fixture, plus {name: chunk index}."""
    m = GFSLModel(N, key_range, cap_bottom, cap_upper)
    names = {}
    levels = sorted(spec)
    for l in levels:
        for j, (name, _) in enumerate(spec[l]):
            names[name] = m.head[l] if j == 0 else m.alloc(l)
    for l in levels:
        chunks = spec[l]
        for j, (name, entries) in enumerate(chunks):
            c = names[name]
            ch = m.pool[c]
            ents = []
            if l == 0:
                ks = ([NEG_INF] if j == 0 else []) + [k + 1 for k in entries]
                ents = [E(k, 0 if k == NEG_INF else 1000 + k) for k in ks]
            else:
                for k, target in entries:
                    kk = NEG_INF if k == "-inf" else k + 1
                    ents.append(E(kk, names[target]))
            assert len(ents) <= m.DSIZE
            for i in range(m.DSIZE):
                ch[i] = ents[i] if i < len(ents) else EMPTY
            last = j == len(chunks) - 1
            mx = INF if last else max(e & 0xFFFFFFFF for e in ents)
            ch[m.NEXT] = E(mx, NULL if last else names[chunks[j + 1][0]])
            ch[m.LOCK] = E(FREE, 0)
        real = any(not (isinstance(x, tuple) and x[0] == "-inf") for _, es in chunks for x in es)
        m.counter[l] = len(chunks) if real else 0
    return m, names


def image(m):
    """(meta dict, flat uint64 entries) for gfsl_load."""
    import numpy as np
    ent = np.array([e for ch in m.pool for e in ch], dtype=np.uint64)
    meta = dict(head=list(m.head), counters=list(m.counter), used_bottom=m.bump[0],
                used_upper=m.bump[1], cap_bottom=m.cap_bottom, cap_upper=m.cap_upper,
                chunk_entries=m.N)
    return meta, ent
