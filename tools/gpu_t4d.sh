cd $GRAFT_REPO_ROOT
export MDH_DEBUG_SYNC=1
timeout 400 python -m pytest tests/test_gpu_parity.py -q -k "mcc_bf16 or tcgen05" > gpurun_out/t4d.txt 2>&1
timeout 200 python -c "
import sys; sys.path.insert(0,'tests')
from gpu_util import run_gpu, assert_close_points
from mdh_workloads import specs as S, gen as G
spec=S.matmul(4096,4096,4096,'bf16'); x=G.matmul_inputs(4096,4096,4096,'bf16','signed'); got,p=run_gpu(spec,x,force_tile='cluster=2'); print(p.describe()['t4_variant']); assert_close_points(spec,x,got,1e-2,n=2000); print('cluster2 parity ok')
" >> gpurun_out/t4d.txt 2>&1
unset MDH_DEBUG_SYNC
timeout 300 python tools/time_one.py mcc_bf16 matmul_bf16 >> gpurun_out/t4d.txt 2>&1
timeout 300 python tools/time_one.py matmul_bf16 --force-tile cluster=2 >> gpurun_out/t4d.txt 2>&1
