#!/bin/bash
mkdir -p gpurun_out
cd scripts/probe && DASP_LIB=../../build/libdasp_DASP_EXP_HOT=1.so timeout 1200 python hot_l1.py c3 > ../../gpurun_out/hot_l1.jsonl 2> ../../gpurun_out/hot_l1.err; echo rc=$?; cd ../..
cat gpurun_out/hot_l1.jsonl; tail -3 gpurun_out/hot_l1.err
