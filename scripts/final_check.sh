#!/bin/bash
# End-of-round check on one GPU (outputs in gpurun_out/): the whole -m gpu suite, smoke(),
# the round measurements (scripts/round_measure.sh) and an ncu capture of the cfg2 kernel
# plus the default bench command's launch list (scripts/ncu_captures.sh).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m pytest tests -m gpu -q > gpurun_out/final_gputest.log 2>&1; echo rc=$? >> gpurun_out/final_gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo rc=$? >> gpurun_out/final_smoke.log
bash scripts/round_measure.sh > gpurun_out/final_round.txt 2>&1
bash scripts/ncu_captures.sh cfg2 > gpurun_out/final_ncu.txt 2>&1
