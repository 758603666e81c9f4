import sys; sys.path.insert(0,'.')
import numpy as np, torch, inputs, oracle, paper_conf_sc_munksgaardhso22_b200 as nwb
for n in [1,2,3,5,8,33,100,300,1000]:
    for tile in [0,16]:
        s,r = inputs.make_problem(n,10)
        want = oracle.nw_ref(s.copy(), r, 10)
        S=torch.from_numpy(s).cuda(); R=torch.from_numpy(r).cuda()
        nwb.nw_fill(S,R,10,tile); torch.cuda.synchronize()
        got=S.cpu().numpy()
        bad=np.argwhere(got!=want)
        print(n,tile,len(bad), bad[:3].tolist(), [ (int(got[i,j]),int(want[i,j]), int(r[i,j])) for i,j in bad[:3]])
        if n<=3: print(got); print(want); print(r)
