"""Bank-conflict degree of the scan DFA lookups for several shared-memory layouts (CPU simulation
over 1 MiB of corpus text, 32 lanes x 64-byte spans as the kernel runs them).  Analysis only."""
import numpy as np, sys
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
import inputs
words = inputs.dictionary()
buf, census, _ = inputs.gen_bytes(inputs.SEED_CORPUS, 0, 1<<20, grep_plants=True)
def isw(c): return (97<=c<=122) or (65<=c<=90) or (48<=c<=57) or c==95
# trie
child = [dict(), dict()]; acc=[0,0]
for d,w in enumerate(words):
    if not all(isw(c) for c in w): continue
    s=0
    for c in w:
        if c not in child[s]:
            child[s][c]=len(acc); child.append(dict()); acc.append(0)
        s=child[s][c]
    if not acc[s]: acc[s]=d+1
ns=len(acc); print('trie states', ns)
# lane traces: 32 lanes, span 64, warp tile 2048
n=len(buf)//2048*2048
tab = np.zeros((256, ns+64), dtype=np.int32)
for s in range(ns+64):
    r = 0 if s>=ns else s
    for b in range(256):
        if not isw(b): nx = ns+acc[r]-1 if (r>=2 and acc[r]) else 0
        elif r==1: nx=1
        else: nx = child[r].get(b, 1)
        tab[b,s]=nx
X = np.frombuffer(bytes(buf[:n]),dtype=np.uint8).reshape(-1,32,64)  # tiles, lanes, bytes
T=X.shape[0]
states = np.zeros((T,32,64),dtype=np.int32)
st = np.zeros((T,32),dtype=np.int32)
prev = np.concatenate([np.zeros((T,1),dtype=np.uint8), X[:,:-1,-1]],axis=1)
prev[1:,0]=X[:-1,-1,-1]
vw = np.vectorize(isw)
st[:] = np.where(vw(prev),1,0)
for i in range(64):
    states[:,:,i]=st
    st = tab[X[:,:,i].astype(np.int64), st]
cols = X.astype(np.int64)
def degree(word_addr):
    # word_addr: (T,32,64) 4-byte word addresses; conflict degree = max over banks of distinct addrs
    tot=0
    wa = word_addr.transpose(0,2,1).reshape(-1,32)
    bank = wa % 32
    deg = np.zeros(len(wa))
    for b in range(32):
        m = bank==b
        # distinct addresses per row in bank b
        a = np.where(m, wa, -1)
        a.sort(axis=1)
        d = (np.diff(a,axis=1)!=0) & (a[:,1:]>=0)
        cnt = d.sum(axis=1) + (a[:,0]>=0)
        deg = np.maximum(deg, cnt)
    return deg.mean()
for nsp in [450, 454, 458, 466, 482, 514, 578]:
    wa = (cols*nsp*2 + states*2)//4
    print('transposed nsp', nsp, 'stride words', nsp/2, 'deg', degree(wa))
# state-major: [state][col] with 129 cols
for ncp in [129, 130, 131, 133, 160]:
    wa = (states*ncp*2 + np.minimum(cols,128)*2)//4
    print('state-major ncol', ncp, 'deg', degree(wa))
# u32 entries transposed (one entry per word)
for nsp in [449, 451, 455]:
    wa = (cols*nsp + states)
    print('u32 transposed nsp', nsp, 'deg', degree(wa))
