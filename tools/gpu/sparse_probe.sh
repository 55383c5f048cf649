# tcgen05.mma.sp metadata layout probe (tools/gpu/exp/sparse_probe.cu, built with -cudart shared):
# decodes which TMEM lane and nibble supply the 2:4 pattern of each (row, K group)
cd tools/gpu/exp
for args in "1 2 0" "2 2 0" "2 -1 0"; do timeout 60 ./sparse_probe $args; done
