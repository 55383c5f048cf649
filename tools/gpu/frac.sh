# L2 policy of the gathered rows at G = 1, 4, 8: the adaptive default vs forced evict_first / evict_last
bash tools/gpu/abe.sh "PSIM_NONE=0 PSIM_ROW_POLICY=first PSIM_ROW_POLICY=last"
