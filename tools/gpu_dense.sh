#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-dense}; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x > $O/gpu_pytest.log 2>&1; echo "rc=$?" >> $O/gpu_pytest.log
LV_TRACE=1 timeout 300 python -c "
import sys; sys.path.insert(0,'tests')
import test_gpu_parity as t, paper_conf_ipps_naimmht17_b200 as lv
for name in ['rmat15','lfr5k','hubs','giant_hub']:
    g=t.GRAPHS[name](); lv.Graph.from_csr(g.rowptr,g.col,g.w).run(lv.params())
" > /dev/null 2> $O/small_trace.err
bash tools/gpu_abn.sh $1_ab base tree
