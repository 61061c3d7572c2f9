#!/bin/bash
# step-by-step slated smoke test with short timeouts (development aid)
EP=/slate-smoke-$$
SLATE_DEBUG=1 ./paper_conf_ipps_allenf019_b200/bin/slated --endpoint $EP > gpurun_out/slated.log 2>&1 &
D=$!
sleep 8
echo "--- attach"
timeout 30 python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_allenf019_b200 import slate as S
s=S.Session('$EP'); print('info', s.info()); s.close(); print('closed')
" 2>&1 | tail -5
echo "--- client"
timeout 60 python tests/ipc_client.py $EP triad 301 2>&1 | tail -8
echo "--- daemon log"
kill -TERM $D; sleep 2; kill -9 $D 2>/dev/null
tail -40 gpurun_out/slated.log
