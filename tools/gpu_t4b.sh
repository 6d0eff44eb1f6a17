cd $GRAFT_REPO_ROOT
export MDH_DEBUG_SYNC=1
timeout 60 python -c "
import sys; sys.path.insert(0,'tests')
from gpu_util import run_gpu, assert_close_points
from mdh_workloads import specs as S, gen as G
for M,N,K in [(512,512,512),(1024,1024,1024),(4096,4096,4096)]:
    spec=S.matmul(M,N,K,'bf16'); x=G.matmul_inputs(M,N,K,'bf16','ones'); got,p=run_gpu(spec,x); print(M,N,K,p.describe()['t4_variant'], float(got[0].min()), float(got[0].max()), flush=True)
" > gpurun_out/t4c.txt 2>&1
echo "rc=$?" >> gpurun_out/t4c.txt
timeout 400 python -m pytest tests/test_gpu_parity.py -q -k "tcgen05 or bf16" >> gpurun_out/t4c.txt 2>&1
unset MDH_DEBUG_SYNC
timeout 300 python tools/time_one.py matmul_bf16 >> gpurun_out/t4c.txt 2>&1
timeout 300 python tools/time_one.py matmul_bf16 --force-tile cluster=1 >> gpurun_out/t4c.txt 2>&1
