# Full-batch parity evidence on the GPU box (one gpurun call, ~45 min of oracle time for C5):
#   gpurun --timeout 4000 -- bash tools/run_full_parity.sh
# writes gpurun_out/full_parity_C3.json, gpurun_out/full_parity_C5.json and the logs.
set -x
python -c "import __graft_entry__ as g; g.build()"
python tests/full_parity.py 3 > gpurun_out/full_parity_C3.log 2>&1
python tests/full_parity.py 5 > gpurun_out/full_parity_C5.log 2>&1
