for zp in 3 1 0; do
HYDRO_ZPROMO=$zp timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_zone_stage -s 2 -c 1 --csv python tools/prof_run.py sedov512 3 2>/dev/null | grep -E "dram|duration" | awk -F'","' -v zp=$zp '{print "ZPROMO=" zp, $(NF-2), $(NF-1), $NF}'
done
