"""Host estimate (NumPy, exact int64 distances) of how many rows a one-partition search epilogue
could not decide: the ratio test is only provably failed when d1 >= 0.64 * (best distance outside the
winning group of G columns).  Prints the pass rate and the undecided rate for G = 64 .. 4 on a sample
of the synthetic workload (12 queries x 300 references)."""
import numpy as np, sys
sys.path.insert(0,'.')
import tidgen
R=300; B=12
refs,_=tidgen.refs(0,R,256)
qs,_=tidgen.queries(0,B,1000,R_total=R,m=256)
q=qs.reshape(-1,128).astype(np.int64)    # (B*1000,128)
r=refs.reshape(-1,128).astype(np.int64)  # (R*256,128)
nq=(q*q).sum(1); nr=(r*r).sum(1)
tot=0; res={}
for rb in range(0,R,50):
    rr=r[rb*256:(rb+50)*256]
    d=nq[:,None]+nr[None,rb*256:(rb+50)*256]-2*(q@rr.T)   # (n, 50*256)
    d=d.reshape(len(q),50,256)
    s=np.sort(d,axis=2)
    d1=s[:,:,0]; d2=s[:,:,1]
    passed=(25*d1<16*d2)
    res.setdefault('pass',0); res['pass']+=passed.sum()
    am=np.argmin(d,axis=2)
    for G in (64,32,16,8,4):
        g=am//G
        dd=d.reshape(len(q),50,256//G,G)
        gm=dd.min(axis=3)  # group minima
        # d2_T = min over groups other than winner's
        gm2=gm.copy()
        np.put_along_axis(gm2,g[...,None],np.iinfo(np.int64).max,axis=2)
        dT=gm2.min(axis=2)
        unc=(25*d1<16*dT)   # not provably failing
        res.setdefault(G,0); res[G]+=unc.sum()
    tot+=d1.size
print('rows',tot,'pass rate',res['pass']/tot)
for G in (64,32,16,8,4): print('group',G,'uncertain',res[G]/tot)
