"""Pure-Python brute force for tiny inputs (test infrastructure).

These are deliberately *different constructions* from oracle.c: they scan all
edges of the COO (never a CSR), use Python's stable `sorted`, dicts, and the
paper's own listing code run in PyTorch, so that a mistake in the oracle's
construction cannot be reproduced here by retyping.
"""
from __future__ import annotations

import numpy as np


def tcsr_by_scanning(num_nodes, src, dst, t, undirected=True):
    """Per node: walk the COO in edge order, collect incident entries, stable-sort by t."""
    per_node = []
    for v in range(num_nodes):
        ent = []
        for e in range(len(src)):
            if int(src[e]) == v:
                ent.append((float(t[e]), e, int(dst[e])))
            if undirected and int(dst[e]) == v:
                ent.append((float(t[e]), e, int(src[e])))
        ent = sorted(ent, key=lambda x: x[0])  # stable: keeps (eid, fwd-before-rev) order
        per_node.append(ent)
    indptr = np.zeros(num_nodes + 1, np.int64)
    for v in range(num_nodes):
        indptr[v + 1] = indptr[v] + len(per_node[v])
    nbr = np.array([x[2] for ent in per_node for x in ent], np.int32)
    eid = np.array([x[1] for ent in per_node for x in ent], np.int32)
    ts = np.array([x[0] for ent in per_node for x in ent], np.float32)
    return indptr, nbr, eid, ts


def candidates_by_scanning(src, dst, t, v, tq, undirected=True):
    """All (t_e, e, nbr) incident to v with t_e < tq, in (t, eid, fwd-first) order."""
    out = []
    tq = np.float32(tq)
    for e in range(len(src)):
        te = np.float32(t[e])
        if not (te < tq):
            continue
        if int(src[e]) == v:
            out.append((float(te), e, 0, int(dst[e])))
        if undirected and int(dst[e]) == v:
            out.append((float(te), e, 1, int(src[e])))
    out.sort(key=lambda x: (x[0], x[1], x[2]))
    return out


def recent_by_scanning(src, dst, t, v, tq, k, undirected=True):
    c = candidates_by_scanning(src, dst, t, v, tq, undirected)
    pick = c[max(0, len(c) - k):]
    return ([x[3] for x in pick], [x[1] for x in pick], [x[0] for x in pick])


def first_occurrence_unique(keys):
    """Dict-insertion-order unique + inverse."""
    pos = {}
    uniq = []
    inv = []
    for kk in keys:
        if kk not in pos:
            pos[kk] = len(uniq)
            uniq.append(kk)
        inv.append(pos[kk])
    return uniq, inv
