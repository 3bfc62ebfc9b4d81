# usage: scripts/build_variant.sh NAME "-DFLAG=..."  -> exp/libdp_NAME.so (experiment builds; select with DP_LIB=...)
mkdir -p exp
cd paper_conf_pldi_carteylm12_b200/csrc
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared $2 -I../../include -I. *.cu *.cpp -o ../../exp/libdp_$1.so
