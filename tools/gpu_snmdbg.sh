cd $GRAFT_REPO_ROOT
python __graft_entry__.py > gpurun_out/build.log 2>&1
for v in auto 2562; do
  if [ $v = auto ]; then unset FFSVA_K1_NT; else export FFSVA_K1_NT=$v; fi
  timeout 300 python bench.py --config snm --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/snmdbg_$v.json 2> gpurun_out/snmdbg_$v.err; echo "$v rc=$?"; tail -2 gpurun_out/snmdbg_$v.err
done
unset FFSVA_K1_NT
CUDA_LAUNCH_BLOCKING=1 timeout 300 python - <<'P' 2>&1 | tail -5
import torch, sys
sys.path.insert(0,'.')
import paper_conf_icpp_zhangcjzly18_b200 as ff
from synth import synth
dev=torch.device('cuda:0'); ctx=ff.Context(dev)
v=synth.Video(seed=1006,width=128,height=100,period=300,on_len=30)
st=ctx.open_stream(width=128,height=100,delta_diff=0.0)
st.set_reference(torch.from_numpy(synth.frames(v,[0],[0],ref=True)).to(dev)); st.snm_load(synth.snm_weights(1006,0))
for n in (4, 1000, 65535, 65536):
    d=torch.from_numpy(synth.frames(v,[0]*4,[0,1,2,3])).to(dev)
    items=[(st, d[i%4], i) for i in range(n)]
    try:
        r=ctx.filter_batch(items); print(n, 'ok', int(r['sdd_pass'].sum()))
    except Exception as e: print(n, 'ERR', e)
P
