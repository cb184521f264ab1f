import os, sys, json, statistics
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_icde_zeng0fcpcwg23_b200 as flb
def timed(fn, reps=3):
    fn(); torch.cuda.synchronize(); ts=[]
    for _ in range(reps):
        s,e=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e)/1e3)
    return statistics.median(ts)
out={}
for bits,count in ((2048,133160),(1024,133160),(3072,16384),(4096,16384)):
    pub, priv = flb.keygen(bits, 0xF1B0+bits)
    g=torch.Generator().manual_seed(1)
    m=torch.randint(-2**31,2**31-1,(count,bits//32),generator=g,dtype=torch.int32); m[:,-1]=0; m=m.cuda()
    for tc in ("1","0"):
        os.environ["FLB_TC"]=tc
        out["%d_pub_enc_tc%s_per_s"%(bits,tc)]=round(count/timed(lambda: flb.encrypt(pub,m,seed=3)))
        if bits>=3072 or bits==1024:
            c=flb.encrypt_crt(priv,m,seed=3)
            out["%d_dec_tc%s_per_s"%(bits,tc)]=round(count/timed(lambda: flb.decrypt(priv,c)))
            out["%d_kh_enc_tc%s_per_s"%(bits,tc)]=round(count/timed(lambda: flb.encrypt_crt(priv,m,seed=3)))
    print(json.dumps(out), flush=True)
