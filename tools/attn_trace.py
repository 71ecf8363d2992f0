import os,sys
sys.path.insert(0,'.')
import torch
from paper_conf_ppopp_liultj25_b200 import _lib
L=_lib.lib()
B,s,nh,dh=4,2048,16,128; h=nh*dh
qkv=torch.randn(B*s,3*h,device='cuda').bfloat16(); O=torch.empty(B*s,h,device='cuda',dtype=torch.bfloat16)
lse=torch.empty(nh,B*s,device='cuda'); dO=torch.randn(B*s,h,device='cuda').bfloat16()
dq=torch.empty(B*s,3*h,device='cuda',dtype=torch.bfloat16); scr=torch.empty(nh,B*s,device='cuda')
L.mario_k_attn_fwd(qkv.data_ptr(),O.data_ptr(),lse.data_ptr(),B,s,nh,dh,1,None)
os.environ['MARIO_ATTN_TC_ONLY']='dkdv'
for i in range(3): L.mario_k_attn_bwd(qkv.data_ptr(),O.data_ptr(),dO.data_ptr(),lse.data_ptr(),dq.data_ptr(),scr.data_ptr(),B,s,nh,dh,1,None)
torch.cuda.synchronize()
os.environ['MARIO_ATTN_TRACE']='1'
L.mario_k_attn_bwd(qkv.data_ptr(),O.data_ptr(),dO.data_ptr(),lse.data_ptr(),dq.data_ptr(),scr.data_ptr(),B,s,nh,dh,1,None)
torch.cuda.synchronize()
