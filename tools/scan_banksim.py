"""Bank-conflict simulation of the byte DFA's shared-memory lookups on the synthetic corpus.

32 lanes scan contiguous 64-byte spans of each 2 KiB warp tile, as scan_range does; for each of
the 64 lookup steps the shared wavefronts of the warp's LDS are max over banks of the distinct
32-bit words requested.  Compares the transposed layout of csrc/scan_core.cuh with a variant that
gives every lane a private copy of the ROOT/DEAD rows in its own bank.  CPU only.
"""
import sys, numpy as np
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs
words = inputs.dictionary()
buf, _, _ = inputs.gen_bytes(1, 0, 1 << 22)
buf = np.frombuffer(bytes(buf), dtype=np.uint8) if not isinstance(buf, np.ndarray) else buf
isw = np.zeros(256, bool)
for c in b'abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789_': isw[c] = True
# trie
child = [dict(), dict()]; acc = [0, 0]
for d, w in enumerate(words):
    s = 0
    for ch in w:
        if ch not in child[s]:
            child[s][ch] = len(acc); child.append(dict()); acc.append(0)
        s = child[s][ch]
    if not acc[s]: acc[s] = d + 1
ns = len(acc); nt = ns + len(words)
nsp = nt
while nsp % 4 != 2: nsp += 1
def col(b): return min(max(b - 47, 0), 76)
T = np.zeros((256, nt), np.int32)
for b in range(256):
    for s in range(nt):
        r = 0 if s >= ns else s
        if not isw[b]: nxt = ns + acc[r] - 1 if (r >= 2 and acc[r]) else 0
        elif r == 1: nxt = 1
        else: nxt = child[r].get(b, 1)
        T[b, s] = nxt
print('states', ns, 'nt', nt, 'nsp', nsp)
# run 32 lanes over spans; record (state before lookup, byte)
N = len(buf) // 2048 * 2048
tiles = buf[:N].reshape(-1, 32, 64)
ntile = tiles.shape[0]
st = np.zeros((ntile, 32), np.int32)
wf_cur = 0; wf_priv = 0; nlook = 0; rootdead = 0
strideb = 2 * nsp
for i in range(64):
    b = tiles[:, :, i].astype(np.int32)
    c = np.clip(b - 47, 0, 76)   # the narrow column map
    # current layout: word = (c*strideb + 2*st)//4
    word = (c * strideb + 2 * st) // 4
    bank = word % 32
    # wavefronts per tile = max over banks of distinct words
    # vectorised: for each tile, count distinct (bank, word) then max per bank
    key = bank.astype(np.int64) * (1 << 32) + word
    ks = np.sort(key, axis=1)
    uniq = np.concatenate([np.ones((ntile, 1), bool), ks[:, 1:] != ks[:, :-1]], axis=1)
    bk = (ks >> 32)
    cnt = np.zeros((ntile, 32), np.int32)
    np.add.at(cnt, (np.repeat(np.arange(ntile), 32)[uniq.ravel()], bk.ravel()[uniq.ravel()]), 1)
    wf_cur += cnt.max(axis=1).sum()
    # private ROOT/DEAD (+emission) rows: lane l's copy in bank l (no conflict among them)
    rd = (st <= 1) | (st >= ns)
    rootdead += rd.sum()
    word2 = np.where(rd, -1 - np.arange(32)[None, :] - 32 * c, word)   # distinct word per lane
    bank2 = np.where(rd, np.arange(32)[None, :], bank)
    key = bank2.astype(np.int64) * (1 << 32) + (word2 + (1 << 20))
    ks = np.sort(key, axis=1)
    uniq = np.concatenate([np.ones((ntile, 1), bool), ks[:, 1:] != ks[:, :-1]], axis=1)
    bk = (ks >> 32)
    cnt = np.zeros((ntile, 32), np.int32)
    np.add.at(cnt, (np.repeat(np.arange(ntile), 32)[uniq.ravel()], bk.ravel()[uniq.ravel()]), 1)
    wf_priv += cnt.max(axis=1).sum()
    nlook += ntile
    st = T[b, st]
print('warp lookups', nlook, 'wavefronts/lookup current %.2f private-rootdead %.2f; root/dead/emit frac %.2f' % (wf_cur / nlook, wf_priv / nlook, rootdead / nlook / 32))
