mkdir -p gpurun_out
cat > /tmp/seg.py <<'PY'
import sys; sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import numpy as np, gen, paper_conf_cluster_zhangzb11a_b200 as gpa
txs = [[1,2,3,4,5],[2,3,4,5,6],[3,4,6,7],[1,3,4,5,6]]
ds = gen.from_lists(txs, 8)
for theta in (1,2,3,4):
    for kern in (0,1,2,4):
        print("theta", theta, "kern", kern, flush=True)
        r = gpa.mine(ds, min_count=theta, options=gpa.Options(count_kernel=kern), keep_candidates=True)
        print(len(r.frequent()), flush=True)
PY
timeout 600 cuda-gdb -batch -ex run -ex bt --args python /tmp/seg.py > gpurun_out/gdb.log 2>&1
