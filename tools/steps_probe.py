import sys, json
sys.path.insert(0, '.')
import torch, bench
dev = torch.device('cuda', 0)
pk = bench.peaks(); flush = bench.L2Flush(dev)
for rep in range(3):
    r = bench.run_mdh_workload('matmul_bf16', 20, 5, 1, 0, dev, flush, pk, with_e2e=False, check=False)
    print(json.dumps([round(t*1e6, 1) for t in r['times']]))
