mkdir -p gpurun_out/mb
(timeout 120 ./tools/tmem_microbench; for v in 0 1 2; do timeout 60 ./tools/epi_microbench $v; done) > gpurun_out/mb/tmem.txt 2>&1
cat gpurun_out/mb/tmem.txt
