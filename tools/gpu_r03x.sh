# round-2 batch x: the whole GPU suite on the deadlock-trap build (PLR_DEADLOCK_TRAP: every spin
# loop traps after 2 s at one site) -- no trap may fire
set -x
TAG=${TAG:-r03x}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
PLR_LIB=$L/libplr_b200_trap.so timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_trap.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_trap.log
grep -c "deadlock trap" gpurun_out/${TAG}_pytest_trap.log >> gpurun_out/${TAG}_pytest_trap.log
true
