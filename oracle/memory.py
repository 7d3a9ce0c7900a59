"""TGN memory path -- TEST INFRASTRUCTURE ONLY.

Memory-based TGNNs keep a memory vector s_v per node and a mailbox (eqs 9-11,
P:129-147; the TGN case study, Listings 3-4):

  messages (eq 9, Listing 3 L16-17 / Listing 4 L24): an edge (u, v, t, e) of the batch
      gives u the message [s_u ; s_v ; e_feat(e)] and v the message [s_v ; s_u ; e_feat(e)];
  coalesce(by='latest') (eq 10, Listing 4 L21): per node only its latest message of the
      batch is kept (TGN "only retains the latest message in the batch for each node",
      P:391) -- reading R26: the latest time, ties broken by the later position in the
      order [src messages ; dst messages] (Listing 3's src_mail-then-dst_mail concat);
  mailbox store (Listing 4 L25): mailbox[v] = that message, mail_ts[v] = its edge time;
  memory update (eq 11, Listing 4 L13-17): for the nodes of a block,
      x = [mailbox[v] ; Phi(mail_ts[v] - mem_ts[v])],  s_v' = GRUCell(x, s_v),
      mem_ts[v] = mail_ts[v]   (Phi = cos(omega dt + phi), the R10 fp32 argument).

Everything is fp64 numpy, one node / message at a time in the order above; the GRU cell
is PyTorch's convention (gates r, z, n; W_ih [3d, d_x], W_hh [3d, d]).  Pins
(tests/test_memory_cpu.py): coalesce against a dict scan, the GRU against
torch.nn.GRUCell in fp64, the memory step against a direct recomputation.
"""
from __future__ import annotations

import numpy as np


def messages(mem, src_b, dst_b, eid_b, efeat):
    """[2B, 2 d_mem + d_e] messages: rows [0, B) for the sources, [B, 2B) destinations."""
    mem = np.asarray(mem, np.float64)
    B = len(src_b)
    out = []
    for role in (0, 1):
        for j in range(B):
            me, other = (src_b[j], dst_b[j]) if role == 0 else (dst_b[j], src_b[j])
            ef = np.asarray(efeat[eid_b[j]], np.float64) if efeat is not None else np.zeros(0)
            out.append(np.concatenate([mem[me], mem[other], ef]))
    return np.stack(out) if out else np.zeros((0, 0))


def coalesce_latest(nodes, times):
    """Unique nodes in order of first occurrence, and for each the position of its latest
    message: max time, ties -> the later position (R26)."""
    first, best = {}, {}
    for j, (v, t) in enumerate(zip(nodes, times)):
        v = int(v)
        if v not in first:
            first[v] = j
            best[v] = j
        else:
            b = best[v]
            if not (times[b] > t):                     # t >= best time -> later wins
                best[v] = j
    uniq = sorted(first, key=lambda v: first[v])
    return np.asarray(uniq, np.int32), np.asarray([best[v] for v in uniq], np.int64)


def mailbox_store(mail, mail_ts, mem, src_b, dst_b, t_b, eid_b, efeat):
    """Listing 4 save_raw_msgs: coalesce the batch's 2B messages, store the latest per
    node into mail / mail_ts (in place).  Returns (uniq, pick)."""
    B = len(src_b)
    nodes = np.concatenate([src_b, dst_b]).astype(np.int64)
    times = np.concatenate([t_b, t_b]).astype(np.float32)
    msgs = messages(mem, src_b, dst_b, eid_b, efeat)
    uniq, pick = coalesce_latest(nodes, times)
    for v, j in zip(uniq, pick):
        mail[v] = msgs[j]
        mail_ts[v] = times[j]
    return uniq, pick


def _phi(dt, omega, phi):
    a = (np.float32(dt) * np.asarray(omega, np.float32)).astype(np.float32)
    b = (a + np.asarray(phi, np.float32)).astype(np.float32).astype(np.float64)
    return np.cos(b).astype(np.float32).astype(np.float64)          # R10, as oracle.c


def gru_cell(x, h, W_ih, W_hh, b_ih, b_hh):
    """PyTorch GRUCell: r, z, n gates (rows [0,d), [d,2d), [2d,3d) of the weights)."""
    d = h.shape[-1]
    gi = W_ih @ x + b_ih
    gh = W_hh @ h + b_hh
    sig = lambda a: 1.0 / (1.0 + np.exp(-a))
    r = sig(gi[:d] + gh[:d])
    z = sig(gi[d:2 * d] + gh[d:2 * d])
    n = np.tanh(gi[2 * d:] + r * gh[2 * d:])
    return (1.0 - z) * n + z * h


def memory_update(mem, mem_ts, mail, mail_ts, nodes, p: dict):
    """Eq 11 for the (unique) nodes, in place: mem[v] = GRUCell([mail[v] ; Phi(dt)], mem[v]),
    dt = fl(mail_ts[v] - mem_ts[v]), mem_ts[v] = mail_ts[v].  Returns the new rows (fp64)."""
    f64 = lambda a: np.asarray(a, np.float64)
    W_ih, W_hh, b_ih, b_hh = f64(p["W_ih"]), f64(p["W_hh"]), f64(p["b_ih"]), f64(p["b_hh"])
    out = []
    for v in nodes:
        v = int(v)
        dt = np.float32(np.float32(mail_ts[v]) - np.float32(mem_ts[v]))
        x = np.concatenate([f64(mail[v]), _phi(dt, p["omega"], p["phi"])])
        h = gru_cell(x, f64(mem[v]), W_ih, W_hh, b_ih, b_hh)
        out.append(h)
    out = np.stack(out) if out else np.zeros((0, mem.shape[1]))
    for v, h in zip(nodes, out):
        mem[int(v)] = h
        mem_ts[int(v)] = mail_ts[int(v)]
    return out
