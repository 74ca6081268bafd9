"""Estimate the DFS steps of the lane join per query under the host planner's
order, and with a closed-form tail of k mutually non-adjacent last nodes
(each attached only to the prefix).  Candidates: label + degree only (a
weaker filter than the bench's L=2 signatures), so the absolute step counts
are upper bounds; the ratios are what this tool is for.
    python tools/tail_sim.py [molecules] [config]"""
import os
import sys
from collections import Counter

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth

n_mol = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
cfg = int(sys.argv[2]) if len(sys.argv) > 2 else 2
Q = synth.config_queries(cfg).graphs()
D = synth.config_data(cfg, count=n_mol).graphs()

freq = Counter()
for labels, _ in D:
    freq.update(labels)


def adjacency(labels, edges):
    adj = [dict() for _ in labels]
    for u, v, b in edges:
        adj[u][v] = b
        adj[v][u] = b
    return adj


def plan(labels, edges):
    n = len(labels)
    adj = adjacency(labels, edges)
    pos = {}
    order = []
    for _ in range(n):
        best, bkey = None, None
        for u in range(n):
            if u in pos:
                continue
            conn = sum(1 for w in adj[u] if w in pos)
            key = (-conn, freq[labels[u]], -len(adj[u]))
            if bkey is None or key < bkey:
                best, bkey = u, key
        pos[best] = len(order)
        order.append(best)
    return order


def connected(nodes, adj):
    nodes = set(nodes)
    if not nodes:
        return True
    st = [next(iter(nodes))]
    seen = {st[0]}
    while st:
        u = st.pop()
        for w in adj[u]:
            if w in nodes and w not in seen:
                seen.add(w)
                st.append(w)
    return seen == nodes


def tail_plan(labels, edges, kmax):
    """order whose last k nodes are mutually non-adjacent, each with a neighbour
    in the (connected) prefix; the largest such k <= kmax (greedy: leaves
    first, then ring nodes whose removal keeps the prefix connected)."""
    n = len(labels)
    adj = adjacency(labels, edges)
    if n < 3:
        return plan(labels, edges), 1
    tail = []
    cand = sorted(range(n), key=lambda u: (len(adj[u]), -freq[labels[u]]))
    for u in cand:
        if len(tail) >= kmax or len(tail) >= n - 1:
            break
        if any(w in adj[u] for w in tail):
            continue
        rest = [x for x in range(n) if x not in tail and x != u]
        if not connected(rest, adj):
            continue
        if not all(any(w in rest for w in adj[t]) for t in tail + [u]):
            continue
        tail.append(u)
    if len(tail) < 2:
        return plan(labels, edges), 1
    rest = [x for x in range(n) if x not in tail]
    sub_l = [labels[x] for x in rest]
    idx = {x: i for i, x in enumerate(rest)}
    sub_e = [(idx[u], idx[v], b) for u, v, b in edges if u in idx and v in idx]
    order = [rest[i] for i in plan(sub_l, sub_e)] + tail
    return order, len(tail)


def suffix_plan(labels, edges, kmax):
    """the planner's order; k = the longest independent suffix (<= kmax)"""
    order = plan(labels, edges)
    adj = adjacency(labels, edges)
    n = len(order)
    k = 1
    while k < min(kmax, n - 1):
        t = order[n - k - 1]
        if any(w in adj[t] for w in order[n - k:]):
            break
        k += 1
    return order, k


def steps(q, g, order, k):
    """DFS steps: partial mappings at depths 0..n-k-1 (each popped once)."""
    ql, qe = q
    dl, de = g
    qa, da = adjacency(ql, qe), adjacency(dl, de)
    n = len(ql)
    cands = [[v for v in range(len(dl)) if dl[v] == ql[u] and len(da[v]) >= len(qa[u])] for u in order]
    pos = {u: i for i, u in enumerate(order)}
    back = [[(pos[w], qa[u][w]) for w in qa[u] if pos[w] < i] for i, u in enumerate(order)]
    total = 0
    last = n - k  # depths [last, n) are the closed-form tail (k == 1: the popc leaf)
    f = [None] * n

    def rec(d, used):
        nonlocal total
        for v in cands[d]:
            if v in used or any(da[v].get(f[j]) != b for j, b in back[d]):
                continue
            f[d] = v
            if d == last - 1:
                total += 1  # the step that computes (and counts) the tail sets
            else:
                total += 1
                rec(d + 1, used | {v})
    if n == 1:
        return 0
    rec(0, frozenset())
    return total


base = tail = 0
rows = []
for qi, q in enumerate(Q):
    o1 = plan(*q)
    o2, k = (tail_plan if os.environ.get('TAIL') == 'greedy' else suffix_plan)(*q, int(os.environ.get('KMAX', 4)))
    s1 = sum(steps(q, g, o1, 1) for g in D)
    s2 = sum(steps(q, g, o2, k) for g in D)
    base += s1
    tail += s2
    rows.append((qi, len(q[0]), k, s1, s2))
for r in sorted(rows, key=lambda r: -r[3])[:25]:
    print(r)
print("steps base", base, "tail", tail, "ratio", tail / max(base, 1))
