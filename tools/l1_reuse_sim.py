"""L1 reuse of the PageRank cold gathers (profiles/pr_floor_r02.md): replays one SM's
gather stream of the seg layout on cfg2 (R-MAT s22 ef16) through a fully associative LRU of
128-byte lines (default 800 lines ~ the ~100 KB of L1 left beside the 128 KB hot table), for the
current tile assignment (strided: 32 consecutive tiles per round, rounds 148*32 tiles apart)
and a contiguous one (each SM owns one contiguous tile range). Usage: l1_reuse_sim.py [sm] [lines]"""
import numpy as np, sys, os, collections
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import grgen
g = grgen.rmat(22, 16, seed=2)
n = g.n
order = np.lexsort((g.src, g.dst))
src = g.src[order]; dst = g.dst[order]
indeg = np.bincount(dst, minlength=n)
outdeg = np.bincount(g.src, minlength=n)
hot = np.zeros(n, bool); hot[np.argsort(-outdeg, kind="stable")[:32768]] = True
# items: per row max(indeg,1); empty rows -> -1
items_per_row = np.maximum(indeg, 1)
off = np.concatenate([[0], np.cumsum(items_per_row)])
items = np.full(off[-1], -1, np.int64)
roff = np.concatenate([[0], np.cumsum(indeg)])
# place sources
pos = off[dst] + (np.arange(len(dst)) - roff[dst])
items[pos] = src
T = (len(items) + 255) // 256
items = np.concatenate([items, np.full(T * 256 - len(items), -1)])
tiles = items.reshape(T, 256)
SM = 148
def sim(tile_seq, cap_lines):
    # tile_seq: list of tile-index lists processed concurrently per round (32 warps)
    lru = collections.OrderedDict()
    acc = miss = 0
    for round_tiles in tile_seq:
        blk = tiles[round_tiles]           # [w, 256]
        # lane L owns 8L..8L+7; instruction k: items 8L+k; interleave over warps
        for k in range(8):
            sl = blk[:, k::8]              # [w, 32]
            for w in range(sl.shape[0]):
                s = sl[w]
                s = s[(s >= 0)]
                s = s[~hot[s]]
                for line in np.unique(s >> 5):
                    acc += 1
                    if line in lru:
                        lru.move_to_end(line)
                    else:
                        miss += 1
                        lru[line] = 1
                        if len(lru) > cap_lines: lru.popitem(last=False)
    return acc, miss
b = int(sys.argv[1]) if len(sys.argv) > 1 else 7
cap = int(sys.argv[2]) if len(sys.argv) > 2 else 800
rounds = (T + SM * 32 - 1) // (SM * 32)
A = [[t for t in range(b * 32 + r * SM * 32, b * 32 + r * SM * 32 + 32) if t < T] for r in range(rounds)]
per = (T + SM - 1) // SM
base = b * per
B = [[t for t in range(base + r * 32, min(base + r * 32 + 32, base + per, T))] for r in range((per + 31) // 32)]
for name, seq in (("strided", A), ("contiguous", B)):
    acc, miss = sim(seq, cap)
    print(name, "line-requests", acc, "misses", miss, "hit%", round(100 * (1 - miss / acc), 1))
