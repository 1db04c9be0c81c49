nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/epi_tc tools/microbench/epi_tc.cu && /tmp/epi_tc
