cd $GRAFT_REPO_ROOT
timeout 300 python - > gpurun_out/r02w_dbg.log 2>&1 <<'PY'
import sys, time, torch
sys.path.insert(0, '.')
import bench
from paper_conf_icde_zhaotl20_b200 import song
from workloads.synth import CONFIGS, make_data
cfg = CONFIGS['glove200']
x, q = make_data(cfg, device='cuda')
t = time.time(); ip = song.build_graph(x, 32, 'ip'); torch.cuda.synchronize(); print('ip', time.time() - t, flush=True)
t = time.time(); cos = song.build_graph_batched(x, 32, 'cosine', prefix=1 << 16, queue_len=128, batch_shift=2); torch.cuda.synchronize(); print('cos', time.time() - t, flush=True)
t = time.time(); adj = song.merge_graph_rows(ip, cos, 8); torch.cuda.synchronize(); print('merge', time.time() - t, flush=True)
print(adj[:3].cpu().numpy(), flush=True)
idx = song.SongIndex(x, adj, metric='ip')
for L in (10, 64, 144, 224, 512):
    t = time.time(); ids, _ = idx.search(q, params=song.Params(K=10, queue_len=L)); torch.cuda.synchronize(); print('L', L, time.time() - t, flush=True)
PY
echo rc=$?
