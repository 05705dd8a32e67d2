./tools/micro/xface2
./tools/micro/xface2 32
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum -k regex:xface --clock-control none ./tools/micro/xface2 2>&1 | grep -E "xface|dram__|duration|lts__" | head -80
