import sys; sys.path.insert(0,'.')
import numpy as np, torch, gen
from oracle import mlp
from paper_conf_sigmod_nakandalak20_b200 import Vista
sys.path.insert(0,'tests')
from test_gpu_mlp import gpu_rows
n,d_s=300,8
tab=gen.make_tables(n,d_s)
v=Vista(0,layers=[0,1],n_str_rows=n,d_s=d_s,n_images_local=n,iters=2,split_seed=5,weight_seed=11)
v.transfer(tab.images,tab.img_keys,tab.X,tab.str_keys,tab.labels)
X,y,te=gpu_rows(v,0)
for it in (1,2,5):
    P,met=v.train_mlp(0,X.shape[1],iters=it,lr=0.01,seed=21)
    P0=mlp.init_params(21,X.shape[1])
    R,L,rm=mlp.train(X,y,te,seed=21,iters=it,lr=0.01)
    print("iters",it,"gpu loss",np.array(met["loss"]),"ref",L)
    for k in ("W1","b1","W2","b2","w3"):
        g=(P[k]-P0[k]); r=(R[k]-P0[k])
        print(k, np.linalg.norm(g-r)/np.linalg.norm(r), np.linalg.norm(g)/np.linalg.norm(r), float(np.dot(g.ravel(),r.ravel())/np.linalg.norm(g)/np.linalg.norm(r)))
    print("b3", P["b3"], R["b3"])
# forward check with initial weights
Xtr=X[~te]
h1,h2,z=mlp.forward(P0,Xtr)
print("h1 mean",h1.mean(),"h2 mean",h2.mean(),"z std",z.std(), "n_train", Xtr.shape)
