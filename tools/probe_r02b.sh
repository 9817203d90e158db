O=gpurun_out/r02b; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_async.py -x -q > $O/async.log 2>&1; echo "rc=$?" >> $O/async.log
for sw in 0 32 64; do
  if [ $sw = 0 ]; then unset VS_SPLIT_WARPS; else export VS_SPLIT_WARPS=$sw; fi
  timeout 300 python tools/spot_scaling.py --config medium --spots 500,250,125,63,32,8,1 > $O/scal_medium_sw$sw.json 2>&1
done
unset VS_SPLIT_WARPS
cat > /tmp/one.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
prob = synth.make_problem("medium")
g = vs.Context.from_problem(prob, vs.score_params())
mp = vs.mh_preset(3, population=256, generations=2)
g.run(mp, 1, np.arange(8, dtype=np.int32))
torch.cuda.synchronize()
PY
VS_GRAPHS=0 timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_8spots.csv python /tmp/one.py > $O/ncu1.log 2>&1
ls $O
