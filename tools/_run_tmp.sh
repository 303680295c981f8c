set -u
g++ -O3 -std=c++17 -pthread -Iinclude tools/aorder_bench.cpp -o /tmp/ab_new && g++ -O3 -std=c++17 -pthread -Iinclude -Itools tools/_aorder_bench_prev.cpp -o /tmp/ab_prev && python tools/dump_od.py 4 degree /tmp/od4.u32
nproc; uptime
for i in 1 2 3; do echo new; TC_AORDER_TRACE=1 /tmp/ab_new /tmp/od4.u32 3 2>&1 | grep aorder | tail -2; echo prev; TC_AORDER_TRACE=1 /tmp/ab_prev /tmp/od4.u32 3 2>&1 | grep aorder | tail -2; done
