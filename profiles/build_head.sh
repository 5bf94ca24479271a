#!/bin/bash
# Build the committed HEAD's libigd into variants/libigd_head.so (A/B baseline for run_variants.sh)
rm -rf /tmp/headsrc && mkdir -p /tmp/headsrc && git archive HEAD paper_conf_sosp_kamathb21_b200/csrc include | tar -x -C /tmp/headsrc
(cd /tmp/headsrc/paper_conf_sosp_kamathb21_b200/csrc && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
  -Xcompiler -fPIC -shared -o "$OLDPWD/variants/libigd_head.so" igd.cu 2>&1 | grep -i " error")
ls -la variants/libigd_head.so
