# compute-sanitizer over the GPU parity tests (small sizes; the full-size and
# > 2^31-element cases, the two-process IPC test and the 10 s peer time-out
# test are left out).  memcheck: out-of-bounds / misaligned global+shared
# accesses; racecheck: shared-memory hazards (COL/ROW cross-warp combines,
# TMA transpose staging, cluster DSMEM combine); synccheck: illegal barriers;
# initcheck: reads of uninitialised global memory.
set -x
export PYTHONUNBUFFERED=1
K='not full_size and not past_2p31 and not absent_rank and not two_processes and not run_host'
T="tests/test_parity_gpu.py tests/test_n4_ops.py tests/test_n3_recurrence.py tests/test_peer.py tests/test_repeat_runs.py tests/test_run_many.py tests/test_edge_cases.py tests/test_odd_gpu.py tests/test_int_gpu.py tests/test_transcendental_gpu.py"
# racecheck and synccheck serialise kernels: the simulated multi-rank peer
# tests (W kernels on W streams waiting for each other's pushes) then report
# their time-out flag by design, so those run under memcheck/initcheck only
KS="$K and not simulated_ranks and not ragged_finalize and not epoch_turnover"
for tool in ${SAN_TOOLS:-memcheck racecheck synccheck initcheck}; do
  k="$K"; case $tool in racecheck|synccheck) k="$KS";; esac
  timeout ${SAN_TIMEOUT:-1200} compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 99 \
    python -m pytest $T -m gpu -q -x -k "$k" -p no:cacheprovider > gpurun_out/san_$tool.log 2>&1
  echo $tool=$?
  grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/san_$tool.log | tail -3
done
