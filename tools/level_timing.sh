# per-level timing of the global phase for one C4 batch of 37 trees (second fit; first is warm-up)
BF_LEVEL_TIMING=1 BF_FIT_TIMING=1 timeout 300 python -c "
import sys; sys.path.insert(0,'.')
import torch, paper_conf_ipps_madougouvln16_b200 as bf
from paper_conf_ipps_madougouvln16_b200 import synthetic as S
X,y,c=S.dataset('C4'); Xd=torch.from_numpy(X).cuda(); yd=torch.from_numpy(y).cuda()
bf.fit(Xd,yd,ntree=37,seed=1,trees_in_flight=37).free(); torch.cuda.synchronize()
print('=====', file=sys.stderr)
bf.fit(Xd,yd,ntree=37,seed=1,trees_in_flight=37).free(); torch.cuda.synchronize()
" 2>&1 | sed -n '/=====/,$p' | python -c "
import sys,re
sc=pa=0; n=0
for l in sys.stdin:
    m=re.search(r'scan=([0-9.]+) mid=([0-9.]+) part=([0-9.]+)', l)
    if m: sc+=float(m.group(1)); pa+=float(m.group(3)); n+=1
    if m: print(l.strip()[:150])
    if 'fit timing' in l: print(l.strip())
print('levels',n,'scan total %.1f ms  part total %.1f ms'%(sc,pa))
"
