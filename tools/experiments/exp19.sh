#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
# sanitizer pass on small shapes, every kernel family
for args in '[16,16,16,16] [3,2,1,0] 8' '[16,16,16,16] [1,0,3,2] 8' '[16,16,16,16] [0,2,3,1] 8' '[3,64,96] [0,2,1] 4' '[4,358,538] [2,1,0] 4' '[16,16,16,16,16,16] [1,0,2,4,3,5] 8' '[5,130,77] [1,0,2] 4'; do
  set -- $args
  for h in '{}' '{"variant":1}' '{"variant":2}'; do
    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/repro.py "$1" "$2" "$3" "$h" > gpurun_out/san.log 2>&1 || { echo "SANITIZER FAIL $args $h"; tail -20 gpurun_out/san.log; }
    compute-sanitizer --tool racecheck --error-exitcode 9 python tools/repro.py "$1" "$2" "$3" "$h" > gpurun_out/race.log 2>&1 || { echo "RACECHECK FAIL $args $h"; tail -20 gpurun_out/race.log; }
  done
done > gpurun_out/sanitizer.txt 2>&1
echo "sanitizer done" >> gpurun_out/sanitizer.txt
