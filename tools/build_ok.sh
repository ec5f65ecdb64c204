#!/bin/bash
# build libgbdt.so; non-zero exit and the errors if anything fails
cd /root/repo/paper_conf_ipps_wenhkls18_b200/csrc && make -s -j8 2>&1 | grep -E "error" && exit 1
cd /root/repo/paper_conf_ipps_wenhkls18_b200/csrc && make -s -j8 >/dev/null 2>&1 || { make 2>&1 | tail -20; exit 1; }
echo build-ok
