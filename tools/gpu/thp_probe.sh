# host-side probe: THP settings and the random-row gather rate with / without THP (tools/cpu_gather_bench.cpp)
cat /sys/kernel/mm/transparent_hugepage/enabled /sys/kernel/mm/transparent_hugepage/defrag /sys/kernel/mm/transparent_hugepage/shmem_enabled 2>&1
g++ -O3 -march=native -pthread -o /tmp/cg tools/cpu_gather_bench.cpp
/tmp/cg 57 512 400000 0
/tmp/cg 57 512 400000 1
