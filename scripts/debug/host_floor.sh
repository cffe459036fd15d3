nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o /tmp/host_floor scripts/debug/host_floor.cu \
  -Lpaper_conf_icdcs_zhaozw24_b200 -ladapcc -Xlinker -rpath=$PWD/paper_conf_icdcs_zhaozw24_b200 && /tmp/host_floor
