"""Numpy emulation (CPU, test of an idea, DESIGN.md R-B5): would storing fp32
populations shifted by f^eq(1, u_ref) (u_ref = inlet velocity) instead of by
the weights w shrink the fp32 drift of a quasi-steady inflow / outflow flow?
Single-level D3Q19 BGK channel 40x21x21, -x velocity inlet (moving-wall
bounce-back), +x outflow (f = w), no-slip y/z walls, omega = 1.99; fp32 in both
representations (the shifted equilibrium evaluated in difference form, every
term small in the free stream) against fp64.  Measured after 200 steps:
err_u 2.55e-6 (w shift) vs 1.96e-6 (u_ref shift), err_rho 5.6e-7 both.
    python tools/fp32_shift_emulation.py [steps=400]
"""
import numpy as np, sys
ex=np.array([0,1,-1,0,0,0,0,1,-1,1,-1,1,-1,1,-1,0,0,0,0]);ey=np.array([0,0,0,1,-1,0,0,1,-1,-1,1,0,0,0,0,1,-1,1,-1]);ez=np.array([0,0,0,0,0,1,-1,0,0,0,0,1,-1,-1,1,1,-1,-1,1])
w=np.array([1/3]+[1/18]*6+[1/36]*12); Q=19; opp=np.array([0]+[q+1 if q%2 else q-1 for q in range(1,Q)])
def feq(rho,ux,uy,uz):
    eu=ex[:,None,None,None]*ux+ey[:,None,None,None]*uy+ez[:,None,None,None]*uz; usq=ux*ux+uy*uy+uz*uz
    return w[:,None,None,None]*rho*(1+3*eu+4.5*eu*eu-1.5*usq)
def run(dt, shift, steps, n=(40,21,21), uin=0.05, omega=1.99):
    uref=np.array([uin,0,0]) if shift else np.zeros(3)
    one=np.ones((1,1,1)); fref=feq(one,one*uref[0],one*uref[1],one*uref[2])[:,0,0,0]
    nx,ny,nz=n; rho=np.ones(n); ux=np.full(n,uin); uy=np.zeros(n); uz=np.zeros(n)
    g=(feq(rho,ux,uy,uz)-fref[:,None,None,None]).astype(dt)
    fr=fref.astype(np.float64)
    for s in range(steps):
        # collide (in dt)
        f=g  # shifted
        drho=f.sum(0,dtype=dt); jx=(ex[:,None,None,None]*f).sum(0,dtype=dt)+dt(uref[0]); jy=(ey[:,None,None,None]*f).sum(0,dtype=dt); jz=(ez[:,None,None,None]*f).sum(0,dtype=dt)
        rho=dt(1)+drho; ux,uy,uz=jx/rho,jy/rho,jz/rho
        geq=(feq(rho.astype(np.float64),ux.astype(np.float64),uy.astype(np.float64),uz.astype(np.float64))-fr[:,None,None,None]).astype(dt) if dt==np.float64 else None
        if dt==np.float32 and shift:
            jpx=(ex[:,None,None,None]*f).sum(0,dtype=dt); jpy=jy; jpz=jz
            ur=uref.astype(dt)
            ej=ex[:,None,None,None].astype(dt)*jpx+ey[:,None,None,None].astype(dt)*jpy+ez[:,None,None,None].astype(dt)*jpz
            eur=(ex*uref[0]+ey*uref[1]+ez*uref[2]).astype(dt)[:,None,None,None]
            j2=jpx*jpx+jpy*jpy+jpz*jpz; jur=jpx*ur[0]+jpy*ur[1]+jpz*ur[2]; ur2=dt(uref@uref)
            inv=dt(1)/rho
            geq=(w[:,None,None,None].astype(dt)*(drho+dt(3)*ej+(dt(4.5)*(ej*ej+dt(2)*ej*eur-drho*eur*eur)-dt(1.5)*(j2+dt(2)*jur-drho*ur2))*inv)).astype(dt)
        elif dt==np.float32:
            # evaluate feq-fref in fp32 like a kernel would (naively)
            eu=ex[:,None,None,None].astype(dt)*ux+ey[:,None,None,None].astype(dt)*uy+ez[:,None,None,None].astype(dt)*uz
            usq=ux*ux+uy*uy+uz*uz
            geq=(w[:,None,None,None].astype(dt)*(drho+rho*(dt(3)*eu+dt(4.5)*eu*eu-dt(1.5)*usq)) + (w-fref).astype(dt)[:,None,None,None]).astype(dt)
        gs=(dt(1-omega)*g+dt(omega)*geq).astype(dt)
        # stream (pull) with BCs
        gn=np.empty_like(gs)
        for q in range(Q):
            src=np.roll(gs[q],(ex[q],ey[q],ez[q]),axis=(0,1,2))
            # masks of links from outside
            x=np.arange(nx)[:,None,None]-ex[q]; y=np.arange(ny)[None,:,None]-ey[q]; z=np.arange(nz)[None,None,:]-ez[q]
            outy=(y<0)|(y>=ny); outz=(z<0)|(z>=nz); outxl=np.broadcast_to(x<0,n); outxr=np.broadcast_to(x>=nx,n)
            outy=np.broadcast_to(outy,n); outz=np.broadcast_to(outz,n)
            bb=gs[opp[q]]
            c=dt(fref[opp[q]]-fref[q])
            wall=bb+c  # noslip
            inl=bb+c+dt(6*w[q]*ex[q]*uin)
            outf=np.full(n,dt(w[q]-fref[q]))
            v=src
            v=np.where(outxr,outf,v)
            v=np.where(outxl,inl,v)
            v=np.where(outy|outz,wall,v)
            gn[q]=v
        g=gn
    drho=g.sum(0); jx=(ex[:,None,None,None]*g).sum(0)+uref[0]
    return (1+drho).astype(np.float64),(jx/(1+drho)).astype(np.float64)
steps=int(sys.argv[1]) if len(sys.argv)>1 else 400
r64,u64=run(np.float64,False,steps)
r64s,u64s=run(np.float64,True,steps)
print("fp64 shift vs noshift",np.abs(u64s-u64).max()/np.abs(u64).max())
for sh in (False,True):
    r32,u32=run(np.float32,sh,steps)
    print("shift",sh,"err_u",np.abs(u32-u64).max()/np.abs(u64).max(),"err_rho",np.abs(r32-r64).max())
